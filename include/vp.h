/* vp.h — C ABI of libvp.so, a B200 (sm_100a) implementation of the VersaPipe pipeline
 * runtime (Zheng, Oh, Zhai, Shen, Yi, Chen; MICRO-50 2017).
 *
 * Citations "L<n>" are line numbers of the paper text.  The calls follow
 * the paper's programming model: "users only need to write the operations for each
 * pipeline stage. VersaPipe will then automatically assemble the stages into a hybrid
 * execution model and configure it" (L3 abstract; L13 §3; L37 §6).
 *
 * Conventions
 *  - Every call returns vp_status (VP_OK == 0).  No C++ exception crosses the ABI.
 *  - Out-parameters come last.  Handles are opaque and NOT thread-safe (one per host thread).
 *  - Call order is enforced: create -> stage_register (all stages) -> insert ->
 *    configure | autotune -> run (repeatable) -> destroy.  Violations: VP_ERR_INVALID.
 *  - Device pointers are CUDA device addresses on the pipeline's device.  "Borrowed"
 *    pointers must stay valid until vp_pipeline_destroy; "copied" data is copied
 *    before the call returns.
 *  - On any error the detailed message is available from vp_last_error(p).
 */
#ifndef VP_H
#define VP_H
#include <stddef.h>
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

typedef enum vp_status {
  VP_OK = 0,
  VP_ERR_INVALID = 1,        /* bad argument or call order                                  */
  VP_ERR_UNSUPPORTED = 2,    /* e.g. RTC on a recursive / latched group (L11: RTC suits     */
                             /* "regular pipeline programs (without recursion or global     */
                             /* synchronizations)")                                         */
  VP_ERR_CUDA = 3,           /* CUDA runtime error; text in vp_last_error                   */
  VP_ERR_OOM = 4,
  VP_ERR_QUEUE_OVERFLOW = 5, /* a producer found its target ring full for > 200 ms          */
  VP_ERR_TIMEOUT = 6,        /* device watchdog (vp_pipeline_desc.watchdog_ms) or tuner cap */
  VP_ERR_BINDING = 7,        /* strict binding requested and a quota was not reached        */
  VP_ERR_FANOUT = 8          /* a stage emitted more items than its declared fan-out        */
} vp_status;

/* Execution models, §4: RTC, KBK, Megakernel (§4.1), coarse and fine
 * pipeline (§4.2.2), hybrid (§4.2.3). */
typedef enum vp_model {
  VP_RTC = 0,
  VP_KBK = 1,
  VP_MEGAKERNEL = 2,
  VP_COARSE = 3,
  VP_FINE = 4,
  VP_HYBRID = 5,
  /* KBK with its control loop on the device: the same per-stage wave kernels, sized by a
   * planner kernel from the live queue counts and repeated by a CUDA-graph while node until
   * the pipeline drains (no host round trip per wave).  A stronger per-stage-kernel
   * baseline than the paper's host-driven KBK (Fig. 3b, L13: "pipeline logic control is
   * implemented on the CPU side"); SURVEY §8 a11. */
  VP_KBK_GRAPH = 6
} vp_model;

/* Per-group models inside VP_HYBRID (the auto-tuner explores "RTC, KBK, Megakernel,
 * and fine pipeline" per group, L45).  Groups are coarse-pipelined with each other. */
typedef enum vp_group_model {
  VP_GROUP_RTC = 0,
  VP_GROUP_KBK = 1,
  VP_GROUP_MEGA = 2,
  VP_GROUP_FINE = 3
} vp_group_model;

/* Built-in stage functions compiled into libvp.so (BaseStage::execute, L37).  A pipeline
 * registers the stages of ONE workload family, in this order.  User-defined families
 * use the C++ template layer (csrc/vp_runtime.cuh) and are instantiated at build time. */
typedef enum vp_stage_kind {
  VP_KIND_INVALID = 0,
  /* Fig. 9 toy (L37): S1 v*=2, recursive until >= threshold; S2 v+1; S3 sink */
  VP_TOY_S1 = 1, VP_TOY_S2 = 2, VP_TOY_S3 = 3,
  /* Collatz queue stress (not in the paper): step (recursive), sink */
  VP_COLLATZ_STEP = 10, VP_COLLATZ_SINK = 11,
  /* Reyes (Fig. 1, L3; L55): Bound, Split (recursive via Bound), Dice, Shade.  Bound,
   * Split and Dice items (and the seeds vp_insert takes for Bound) are 208-B patches:
   * float x[16], y[16], z[16] (control point P[a][b] at 4a + b, affine: w = 1), then
   * uint32 id = frame << 12 | patch, path, dirs, depth -- the paper's 272-B float4 item
   * (Table 2) without its constant w (reading R-S10).  Shade items are
   * 2032-B grids (vp_stage_kind_info reports every kind's stride).  Register each stage
   * with exactly these strides. */
  VP_REYES_BOUND = 20, VP_REYES_SPLIT = 21, VP_REYES_DICE = 22, VP_REYES_SHADE = 23,
  /* Rasterization (Fig. 16, L59): Vertex + Clip (the paper's Clip), Raster (its
   * Interpolate: triangle -> 8x8 tiles), Fragment (its Shade: coverage + z-buffer) */
  VP_RASTER_VERTEX = 30, VP_RASTER_CLIP = 31, VP_RASTER_RASTER = 32, VP_RASTER_FRAGMENT = 33,
  /* Image pyramid (Fig. 12, L53): Grayscale, HistEq as CDF + Map, Resize (recursive);
   * dependency latches between them */
  VP_PYR_GRAY = 40, VP_PYR_CDF = 41, VP_PYR_MAP = 42, VP_PYR_RESIZE = 43,
  /* CFD (Fig. 15, L55; Rodinia euler3d): Copy, Step Factor, Flux, Time Step; loop of 3 RK
   * steps per outer iteration; tiles of T cells (composite items, L37) */
  VP_CFD_COPY = 50, VP_CFD_STEP_FACTOR = 51, VP_CFD_FLUX = 52, VP_CFD_TIME_STEP = 53,
  /* LBP face detection (Fig. 14, L55): Grayscale, HistEq as CDF + Map, Resize
   * (recursive), Feature Extraction (LBP), Scanning (rows of 24x24 windows) */
  VP_FD_GRAY = 60, VP_FD_CDF = 61, VP_FD_MAP = 62, VP_FD_RESIZE = 63, VP_FD_LBP = 64, VP_FD_SCAN = 65,
  /* Queue microbenchmark (not a paper workload): a self-recursive stage
   * with 4-, 16- or 272-B items (Fig. 9's int; Table 2's window / tile items; the Reyes
   * patch, L61 §8.5), each kind a single-stage pipeline of its own: register one of them.
   * See vp_qbench_params (counters indexed by item size: 0 = 4 B, 1 = 16 B, 2 = 272 B). */
  VP_QB_ITEM4 = 70, VP_QB_ITEM16 = 71, VP_QB_ITEM272 = 72,
  /* the same 4- and 16-B stages built with cluster work stealing (VP_FLAG_CLUSTER_STEAL;
   * SURVEY §8(f-2)): separate kernels, so the plain ones are unchanged */
  VP_QB_ITEM4_CS = 73, VP_QB_ITEM16_CS = 74,
  /* LDPC decoder (Fig. 17, L59): Initialize, C2V, V2C, ProbVar (loops back to C2V for the
   * next of n_iter iterations); items {frame, iteration}; see vp_ldpc_params */
  VP_LDPC_INIT = 80, VP_LDPC_C2V = 81, VP_LDPC_V2C = 82, VP_LDPC_PROBVAR = 83
} vp_stage_kind;

#define VP_MAX_STAGES 8
#define VP_MAX_SM 256

/* vp_pipeline_desc.flags */
#define VP_FLAG_TRACE 0x1u          /* record (stage, item id, smid) of every task           */
#define VP_FLAG_QUEUE_DEPTH 0x2u    /* track max ring depth per stage (one extra read/flush) */
#define VP_FLAG_STRICT_BINDING 0x4u /* vp_run fails with VP_ERR_BINDING on quota shortfall   */
#define VP_FLAG_TIMERS 0x8u         /* in-kernel %globaltimer accumulators per stage/kernel, */
                                    /* and KBK wave times per stage (stage_wave_ms)         */
#define VP_FLAG_ONLINE 0x20u        /* online adaptation (L41-L45): a persistent group whose  */
                                    /* stages can get no more items retires and the host      */
                                    /* relaunches the next group downstream on its SMs         */
                                    /* (persistent plans only; extra grids appear in           */
                                    /* vp_run_stats.kernel_* after the planned ones)           */
#define VP_FLAG_L2_PERSIST 0x40u    /* an L2 access-policy window (persisting) over */
                                    /* every ring's sequence words on the run stream and the  */
                                    /* group streams (sets cudaLimitPersistingL2CacheSize)    */
#define VP_FLAG_SERIALIZE_GROUPS 0x80u /* test hook: each persistent group's grid starts only */
                                      /* after the previous group's grid finished, i.e. what a */
                                      /* profiler's kernel serialisation (or MPS / a co-tenant) */
                                      /* can do to separately launched groups  */
#define VP_FLAG_NO_RERUN 0x100u       /* when the groups of a coarse/fine/hybrid plan cannot all */
                                      /* be resident (a group stalled >= 20 ms on a planned grid */
                                      /* with no resident block), vp_run returns                 */
                                      /* VP_ERR_UNSUPPORTED instead of repeating the run as one  */
                                      /* cooperative megakernel (vp_run_stats.model_rerun)        */
#define VP_FLAG_CLUSTER_STEAL 0x200u  /* a cooperative megakernel of a family   */
                                      /* that allows it (the queue microbenchmark) runs as      */
                                      /* clusters of 2 CTAs, and a CTA with nothing to claim    */
                                      /* takes up to half of its sibling's block-local queue    */
                                      /* over distributed shared memory                         */
                                      /* (vp_run_stats.stolen)                 */
#define VP_FLAG_FULL_RINGS 0x10u    /* persistent plans keep every ring at its registered     */
                                    /* capacity instead of shrinking it to what the producer  */
                                    /* blocks can hold (needed when a recursive stage's live   */
                                    /* frontier is larger, e.g. breadth-first fan-out-2 trees) */

typedef struct vp_pipeline_desc {
  int max_stages;                 /* <= VP_MAX_STAGES                                      */
  uint32_t flags;                 /* VP_FLAG_*                                             */
  int64_t default_queue_capacity; /* ring slots per stage (rounded up to a power of 2);    */
                                  /* 0 = the family's default                              */
  int watchdog_ms;                /* device watchdog per vp_run; 0 = 30000                 */
  int64_t trace_capacity;         /* records, with VP_FLAG_TRACE                           */
} vp_pipeline_desc;

typedef struct vp_stage_desc {
  const char* name;        /* informational, copied                                         */
  int kind;                /* vp_stage_kind                                                 */
  int item_bytes;          /* DataItemType size (L37); must equal the kind's item size      */
  int threads_per_item;    /* threadNum (L37); 0 = the kind's default; informational for    */
                           /* built-ins, whose execute() is written for a fixed mapping     */
  int64_t queue_capacity;  /* ring slots; 0 = pipeline default                              */
  const void* params;      /* HOST pointer to the family's parameter struct (vp_*_params),  */
                           /* copied; the device pointers inside it are BORROWED.  Stages   */
                           /* of one family may repeat it or pass NULL after the first.     */
  size_t params_bytes;     /* sizeof(the vp_*_params struct)                                */
} vp_stage_desc;

/* SM binding / grouping configuration {g, s, b} (L41; Fig. 10 L43). */
typedef struct vp_sm_binding {
  int num_groups;
  int group_of_stage[VP_MAX_STAGES];   /* groups are contiguous stage ranges (L45)           */
  int group_model[VP_MAX_STAGES];      /* vp_group_model, per group                          */
  uint32_t group_sm_mask[VP_MAX_STAGES][VP_MAX_SM / 32]; /* s_flag(group, sm), Fig. 5       */
  int blocks_per_sm[VP_MAX_STAGES];    /* per stage (fine groups) / per group first stage     */
                                       /* (mega/RTC groups); 0 = as many as fit              */
  int batch[VP_MAX_STAGES];            /* items per claim per stage; 0 = default             */
} vp_sm_binding;

typedef struct vp_config {
  int model;                 /* vp_model                                                   */
  int has_binding;
  vp_sm_binding binding;
  int batch;                 /* global items-per-claim override, 0 = per-stage defaults    */
} vp_config;

typedef struct vp_run_stats {
  double device_ms;                         /* CUDA events around the run on the stream   */
  uint64_t dequeued[VP_MAX_STAGES];         /* tasks executed per stage                   */
  uint64_t enqueued[VP_MAX_STAGES];         /* items pushed per stage, seeds included     */
  uint64_t max_depth[VP_MAX_STAGES];        /* with VP_FLAG_QUEUE_DEPTH                   */
  int num_kernels;                          /* persistent kernels launched                */
  int kernel_lo[16], kernel_hi[16];         /* stage range of each persistent kernel      */
  int kernel_quota[16];                     /* requested blocks/SM (0 = fill)             */
  double kernel_ms[16];                     /* CUDA-event duration of each persistent     */
                                            /* kernel on its own stream                   */
  uint32_t blocks_on_sm[16][VP_MAX_SM];     /* blocks that ran the prologue on each SM    */
  uint64_t admitted[16];                    /* blocks that stayed (check_sm/check_sm_blk) */
  uint64_t fallback_admits;                 /* progress-guarantee admissions              */
  uint64_t kbk_launches;                    /* wave launches (KBK / RTC)                   */
  uint64_t trace_records;                   /* with VP_FLAG_TRACE                          */
  int abort_reason;                         /* 0 none, 1 timeout, 2 overflow, 3 fan-out,  */
                                            /* 4 guard, 5 groups not co-resident          */
  int num_sms;
  /* VP_FLAG_TIMERS: block-time (ns, summed over blocks) spent executing each stage     */
  /* (stage-in + execute), publishing its outputs (queue overhead, §8.5), and idle per  */
  /* persistent kernel (no claimable item)                                              */
  uint64_t stage_exec_ns[VP_MAX_STAGES];
  uint64_t stage_flush_ns[VP_MAX_STAGES];
  uint64_t kernel_idle_ns[16];
  /* ring state at the end of the run (diagnostics after an abort): reserved tickets,
   * claimed tickets, published-unclaimed items, seeds claimed; final pending count */
  uint64_t ring_tail[VP_MAX_STAGES], ring_head[VP_MAX_STAGES];
  int64_t ring_count[VP_MAX_STAGES];
  uint64_t seed_head[VP_MAX_STAGES];
  int64_t pending;
  uint64_t kernel_rounds[16];               /* persistent-loop rounds summed over blocks  */
  /* host-driven KBK: summed device time of each stage's wave kernels (every wave uses the
   * whole GPU), i.e. each stage run in isolation -- Table 2's "longest stage" analog (L51) */
  float stage_wave_ms[VP_MAX_STAGES];
  /* the host waited > 2 s for a group's grid to be fully dispatched before launching the
   * next group (SM binding is then not deterministic), per run */
  int dispatch_timeouts;
  /* 1: the planned groups were not co-resident (ABORT_NOT_CORESIDENT), so the run was
   * repeated from its seeds as one cooperative megakernel; device_ms covers both attempts */
  int model_rerun;
  /* family-defined work units per stage (Reyes: micropolygons shaded by the fused
   * [Dice, Shade] chain, i.e. those whose box holds a pixel centre; 0 elsewhere) */
  uint64_t work_units[VP_MAX_STAGES];
  /* VP_FLAG_CLUSTER_STEAL: items taken from a cluster sibling's block-local queue */
  uint64_t stolen[VP_MAX_STAGES];
} vp_run_stats;

typedef struct vp_autotune_opts {
  double time_budget_s;      /* total tuning wall time; 0 = 60 s                           */
  int sm_granularity;        /* SM split step; 0 = 4 (L45 pruning, B200 has 148 SMs)       */
  int batch_choices[4];      /* candidate items-per-claim multipliers; 0-terminated        */
  uint32_t models_allowed;   /* bitmask of 1 << vp_group_model; 0 = all                    */
  int max_candidates;        /* 0 = 400                                                    */
  int repeats;               /* timed runs per candidate (min taken); 0 = 1                */
} vp_autotune_opts;

typedef struct vp_tune_report {
  int candidates_total;      /* after pruning                                              */
  int candidates_run;
  int candidates_timed_out;  /* stopped by timeoutexec (Fig. 10)                           */
  double best_ms;
  double baseline_kbk_ms;
  double baseline_mega_ms;
  int max_blocks_per_sm[VP_MAX_STAGES];  /* profiling component (L13, L45)                */
  int regs_per_thread[VP_MAX_STAGES];
  int smem_per_block[VP_MAX_STAGES];
} vp_tune_report;

/* ---------------- family parameter structs (device pointers are BORROWED) ------------ */
typedef struct vp_toy_params {
  int32_t threshold;         /* THRESHOLD of Fig. 9                                        */
  int32_t pad;
  int32_t* out;              /* sink output values, capacity >= #seeds                     */
  unsigned long long* n_out; /* device counter, reset by every vp_run                      */
} vp_toy_params;

/* Queue microbenchmark.  Item word 0 = id (24 bits) | remaining depth << 24; words 1..
 * = payload id * 2654435761 + k * 40503 (mod 2^32).  A task with fanout > 0 and depth > 0
 * emits `fanout` copies of its item with depth - 1 (whole payload copied); a leaf checks
 * its payload and adds to the per-stage counters.  Tasks per seed: 1 (fan-out 0),
 * depth + 1 (fan-out 1), 2^(depth+1) - 1 (fan-out 2). */
typedef struct vp_qbench_params {
  uint32_t fanout;             /* 0, 1 or 2                                                */
  uint32_t depth;              /* informational (seeds carry their own depth); <= 255      */
  unsigned long long* leaves;  /* [3] leaves per stage (reset by vp_run)                   */
  unsigned long long* idsum;   /* [3] sum of leaf ids per stage                            */
  unsigned long long* bad;     /* [3] leaves whose payload was corrupted                   */
} vp_qbench_params;

/* LDPC decoder (Fig. 17; readings R-L1..R-L6): normalised min-sum on a
 * (dv, dc)-regular parity-check matrix given as edge arrays in check-major order
 * (edge e = m*dc + k joins check m and variable check_vars[e]). */
typedef struct vp_ldpc_params {
  int32_t N, M, dv, dc;        /* variables, checks, degrees (N*dv == M*dc, dc <= 32, dv <= 8) */
  int32_t n_frames, n_iter;    /* frames decoded in one run; iterations per frame              */
  float alpha;                 /* min-sum normalisation                                        */
  int32_t nc_chk, nc_var;      /* items: C2V chunks of the checks, V2C / ProbVar chunks of the */
                               /* variables (1..16 each; reading R-L6)                         */
  int32_t pad;
  const int32_t* check_vars;   /* [M*dc] variable of each edge                                 */
  const int32_t* var_edges;    /* [N*dv] edges of each variable, ascending                     */
  const float* llr;            /* [n_frames*N] channel LLRs                                    */
  float* v2c;                  /* [n_frames*M*dc] work: variable-to-check messages             */
  float* c2v;                  /* [n_frames*M*dc] work: check-to-variable messages             */
  float* post;                 /* [n_frames*N] posterior LLRs after the last iteration         */
  int32_t* errors;             /* [n_frames*n_iter] bits decided 1 per iteration (reset by run) */
  int32_t* latch;              /* [n_frames*2] work: the chunk-join latches (reset by run)      */
} vp_ldpc_params;

typedef struct vp_collatz_params {
  uint32_t* steps_out;       /* [n ids] stopping time per id                               */
  uint32_t* seen;            /* [n ids] times each id reached the sink (reset by vp_run)  */
  uint32_t n_ids;
  uint32_t max_steps;        /* recursion guard                                            */
} vp_collatz_params;

typedef struct vp_reyes_params {
  int32_t W, H, n_frames, patches_per_frame, max_depth;
  int32_t frame_base;        /* item ids carry global frame numbers (id = frame << 12 |    */
                             /* patch); this run renders frames [frame_base, frame_base +   */
                             /* n_frames): M, fb and colour are indexed by frame - frame_base */
                             /* (0 for a whole batch; vp_set_params moves it per chunk)     */
  float t_dice, near_w;
  const float* M;            /* [n_frames][16] view-projection, row-major                  */
  const float* albedo;       /* [patches_per_frame][4]                                     */
  float L[4];                /* light direction                                            */
  void* fb;                  /* [n_frames*H*W] 16-B records {u64 key, f32 s, u32 pad},     */
                             /* reset by vp_run; key = UINT64_MAX when uncovered           */
  float* colour;             /* [n_frames*H*W][4] resolved colour, written by vp_run       */
} vp_reyes_params;

typedef struct vp_raster_params {
  int32_t W, H;
  int64_t n_tris;            /* vertex stage items are triangle ids in [0, n_tris)        */
  const float* M;            /* [16] row-major vertex transform (pixel -> clip)            */
  const float* pos;          /* [n_tris][3][4] vertex positions (x, y, z, w), 16-B aligned */
  const float* col;          /* [n_tris][3][4] vertex colours (r, g, b, -)                  */
  void* setup;               /* [n_tris] x 128 B scratch (per-triangle setup), 128-B aligned */
  unsigned long long* fb;    /* [H*W] depth keys (zkey(z) << 32 | tri), reset by vp_run    */
  float* colour;             /* [H*W][4] resolved colour, written by vp_run                */
  int32_t near_clip;         /* 0: cull triangles with a vertex at w <= 1e-6 (keys carry tri);  */
                             /* 1: clip against z = 0 first (DESIGN R-S9):      */
                             /*    Clip emits 0..2 sub-triangles 2 tri + j, keys carry that id, */
                             /*    setup must hold 2 n_tris records                              */
  int32_t pad0;
  float* ccol;               /* near_clip: [2 n_tris][3][4] sub-triangle vertex colours (scratch, */
                             /* 16-B aligned, written by Clip); ignored when near_clip == 0      */
} vp_raster_params;

typedef struct vp_pyramid_params {
  int32_t S;                 /* image side: power of two in [64, 4096]                     */
  int32_t n_img;             /* Gray items are {img, 0, ty, tx} for the 64x64 tiles        */
  const uint8_t* rgb;        /* [n_img][S][S][3] input, 16-B aligned                       */
  uint8_t* gray;             /* [n_img][S*S] scratch: level-0 grayscale                    */
  uint8_t* pyr;              /* [n_img][stride] output pyramid, levels concatenated;       */
                             /* stride = sum_l (S>>l)^2 rounded up to a multiple of 128    */
  uint32_t* hist;            /* [n_img][256] histograms (reset by vp_run)                  */
  uint8_t* lut;              /* [n_img][256] equalisation LUTs (output)                    */
  int32_t* latch;            /* [n_img][1 + sum_{l>=1} tiles_l^2] dependency latches       */
} vp_pyramid_params;

typedef struct vp_cfd_params {
  int32_t G;                 /* grid side; N = G*G cells                                   */
  int32_t T;                 /* cells per tile item (divides G, multiple of 4)             */
  int32_t n_outer;           /* outer iterations; the final state is vars[(3*n_outer) & 1] */
  int32_t pad0;
  const float* vars0;        /* [5][N] initial state (density, momentum x/y/z, energy)     */
  float* vars;               /* [2][5][N] ping-pong state, 16-B aligned (output)           */
  float* old;                /* [5][N] scratch                                             */
  float* sf;                 /* [N] step factors (scratch)                                 */
  float* flux;               /* [5][N] scratch                                             */
  const float* area;         /* [N]                                                        */
  const int32_t* nb;         /* [4][N] neighbour cell, -1 wall, -2 far field               */
  const float* normals;      /* [4][3][N] face normals                                     */
  float ff[5];               /* far-field conserved state                                  */
  int32_t pad1;
  int32_t* latch;            /* [2][N/T] dependency latches (scratch)                      */
} vp_cfd_params;

typedef struct vp_facedet_params {
  int32_t W, H;              /* level-0 frame size (24 <= W <= 8192, 24 <= H <= 2048)      */
  int32_t n_frames;          /* Gray items are {frame, 0, band, 0}, bands of 32 rows        */
  int32_t n_stages;          /* cascade stages K <= 16                                     */
  int32_t n_weak[16];        /* weak classifiers per stage                                 */
  int32_t thr[16];           /* stage thresholds                                           */
  int32_t n_weak_total;      /* sum(n_weak) <= 128                                         */
  int32_t pad0;
  const uint8_t* rgb;        /* [n_frames][H][W][3]                                         */
  uint8_t* levels;           /* [n_frames][sum_l W_l*H_l] equalised pyramid (scratch/out)  */
  uint8_t* lbp;              /* [n_frames][sum_l W_l*H_l] LBP codes (scratch/out)          */
  uint32_t* hist;            /* [n_frames][256]                                            */
  uint8_t* lut;              /* [n_frames][256]                                            */
  const int32_t* weak;       /* [n_weak_total][12]: cx, cy, mask[8], in, out               */
  uint32_t* det;             /* [det_cap][4] detections {frame, level, x, y}, 16-B aligned */
  unsigned long long* det_count;   /* device counter (reset by vp_run)                     */
  unsigned long long det_cap;
  unsigned long long* survivors;   /* [16] windows passing stage k (reset by vp_run)       */
  unsigned long long* windows;     /* windows evaluated (reset by vp_run)                  */
  int32_t* latch;            /* [n_frames][1 + 3 * sum_l bands_l] dependency latches       */
} vp_facedet_params;

/* ---------------- calls ---------------- */
const char* vp_status_string(vp_status s);
const char* vp_last_error(void* p);

/* Create an empty pipeline on CUDA device `device` (Fig. 2 framework object). */
vp_status vp_pipeline_create(int device, const vp_pipeline_desc* d, void** out);
vp_status vp_pipeline_destroy(void* p);

/* Register the next stage (class Stage_k : public BaseStage, L37).  Stage ids are dense,
 * assigned in registration order; the kinds must be one family in its canonical order. */
vp_status vp_stage_register(void* p, const vp_stage_desc* s, int* stage_id);

/* VersaPipe::insertIntoQueue(initItems, n) (L37).  Items are COPIED (host or device
 * memory per flags) and snapshotted: every vp_run re-seeds from them.  flags:
 *   VP_INSERT_DEVICE  items is a device pointer
 *   VP_INSERT_REPLACE drop previously inserted items of this stage first            */
#define VP_INSERT_DEVICE 0x1
#define VP_INSERT_REPLACE 0x2
vp_status vp_insert(void* p, int stage_id, const void* items, size_t n, int flags);
/* Stream-ordered variant (the copy is enqueued on `cuda_stream`). */
vp_status vp_insert_async(void* p, int stage_id, const void* items, size_t n, int flags, void* cuda_stream);

/* Choose the execution model and SM / block binding (optional step of §6; L37).
 * binding == NULL: defaults (all SMs; coarse: equal SM split; fine: equal block split).
 * batch: items per claim for every stage (0 = per-stage defaults / binding->batch). */
vp_status vp_configure(void* p, int model, const vp_sm_binding* binding, int batch);
vp_status vp_configure_config(void* p, const vp_config* c);
vp_status vp_get_config(void* p, vp_config* out);

/* Run the pipeline to completion on `cuda_stream` (NULL = legacy default stream), then
 * return.  stats may be NULL. */
vp_status vp_run(void* p, void* cuda_stream, vp_run_stats* stats);

/* Device watchdog for subsequent runs, in milliseconds (> 0).  The auto-tuner's
 * timeoutexec(mintime, config) (Fig. 10) uses the same mechanism. */
vp_status vp_set_timeout(void* p, double ms);

/* Offline auto-tuner (L41–L45, Fig. 10): profile, enumerate pruned {g, s, b}, run each
 * candidate under timeoutexec(mintime), keep and apply the fastest.  best/report may be NULL. */
vp_status vp_autotune(void* p, const vp_autotune_opts* o, vp_config* best, vp_tune_report* report);

/* Profiling component (L13, L45): max resident blocks per SM of each single-stage kernel. */
vp_status vp_profile(void* p, int* max_blocks_per_sm, int* regs_per_thread, int* smem_per_block);

/* Change the run-time flags of a pipeline (VP_FLAG_QUEUE_DEPTH, VP_FLAG_STRICT_BINDING,
 * VP_FLAG_TIMERS, VP_FLAG_SERIALIZE_GROUPS, VP_FLAG_NO_RERUN, VP_FLAG_CLUSTER_STEAL; the others are fixed at create
 * and rejected with VP_ERR_INVALID).  old_flags (optional) receives all flags before the change. */
vp_status vp_set_flags(void* p, uint32_t flags, uint32_t* old_flags);

/* Replace the family parameter struct between runs (same family, same params_bytes; it
 * is validated like the one given to vp_stage_register).  E.g. the next chunk of frames of
 * a streamed batch (vp_reyes_params.frame_base, M).  VP_ERR_INVALID on a size mismatch or
 * invalid parameters; the previous parameters then stay in force. */
vp_status vp_set_params(void* p, const void* params, size_t params_bytes);

/* Library-owned / borrowed outputs of the family (sink results). index 0 = primary. */
vp_status vp_get_output(void* p, int index, void** dev_ptr, size_t* bytes);

/* The task trace of the last run (VP_FLAG_TRACE): library-owned device array of 24-B
 * {u64 item id, u32 stage, u32 smid, u32 kernel slot, u32 blockIdx.x} records (the kernel
 * slot indexes vp_run_stats.kernel_*), valid until the next vp_run. */
vp_status vp_get_trace(void* p, void** dev_ptr, size_t* n_records);

vp_status vp_config_to_string(const vp_config* c, char* buf, size_t buf_len);
vp_status vp_config_from_string(const char* s, vp_config* out);

/* Measured ceiling for the L2-atomic rooflines: fire-and-forget 64-bit
 * atomic minimum (the raster z-buffer update) from a full grid to pseudo-random slots of a
 * `slots` x 8-B device buffer; *ops_per_s = n_ops / best-of-3 CUDA-event time.
 * Diagnostics only; it does not touch any pipeline. */
vp_status vp_bench_red_min_u64(int device, unsigned long long slots, unsigned long long n_ops, double* ops_per_s);

/* Item stride (bytes) a built-in stage kind must be registered with (vp_stage_desc.
 * item_bytes), and its threads per item.  VP_ERR_INVALID for an unknown kind.  Host-only:
 * no device is touched. */
vp_status vp_stage_kind_info(int kind, int* item_bytes, int* threads_per_item);

/* Device properties the binding layer needs (no torch types cross the ABI). */
vp_status vp_device_info(int device, int* num_sms, int* cc_major, int* cc_minor);
/* Minimal CUDA plumbing for bindings without their own CUDA runtime. kind: 0 H2D, 1 D2H, 2 D2D */
vp_status vp_memcpy(void* dst, const void* src, size_t bytes, int kind, void* cuda_stream);

#ifdef __cplusplus
}
#endif
#endif

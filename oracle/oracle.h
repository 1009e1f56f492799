/* oracle.h — CPU ORACLE. TEST INFRASTRUCTURE ONLY.
 *
 * Plain, slow, single-threaded C99 implementation of what the VersaPipe hot path
 * computes (PAPER.md = /root/reference/PAPER.md; "L<n>" = its line numbers).  Only
 * tests/, __graft_entry__.smoke() and bench.py's cpu_baseline / --impl reference leg
 * may load this library.  It shares NO code, header, table or constant with the CUDA
 * path in paper_conf_micro_zhengozsyc17_b200/csrc; the two meet only at the seeded
 * input byte layouts produced by paper_conf_micro_zhengozsyc17_b200/inputs.py.
 *
 * Built with gcc -O2 -ffp-contract=off (no FMA contraction, no fast-math, SSE float),
 * SURVEY §8(c-G) rule 2.
 *
 * Two layers per workload (SURVEY §8(c) "Structure"):
 *   1. a *definition* oracle written as the textbook loop/recursion, and
 *   2. the *pipeline* oracle: the generic sequential fixpoint engine below, which
 *      runs each stage's per-item operation over FIFO work queues until every queue is
 *      empty -- the paper's producer/consumer pipeline (L5 §1 "A task of a previous
 *      stage fetches input data from its queue, executes this stage, and finally puts
 *      output data into the queue of the next stage, which is repeated until all stages
 *      finish") executed sequentially.
 */
#ifndef VP_ORACLE_H
#define VP_ORACLE_H
#include <stddef.h>
#include <stdint.h>

#define ORC_MAX_STAGES 8

/* ---------------- generic fixpoint engine (fixpoint.c) ---------------- */
typedef struct orc_fifo {
  uint8_t* data;
  size_t stride, head, tail, cap; /* items [head, tail) are queued */
} orc_fifo;

typedef struct orc_trace_rec { uint64_t id; uint32_t stage, pad; } orc_trace_rec;

struct orc_engine;
typedef void (*orc_exec_fn)(struct orc_engine* e, int stage, const void* item);

typedef struct orc_engine {
  int n_stages;
  orc_fifo q[ORC_MAX_STAGES];
  orc_exec_fn exec;
  void* user;
  uint64_t deq[ORC_MAX_STAGES]; /* items executed per stage                  */
  uint64_t enq[ORC_MAX_STAGES]; /* items pushed per stage (seeds included)   */
  uint64_t max_depth_seen[ORC_MAX_STAGES];
  /* optional trace of (stage, item id) per executed task */
  orc_trace_rec* trace;
  size_t trace_cap, trace_n;
  int error;
} orc_engine;

void orc_engine_init(orc_engine* e, int n_stages, const size_t* strides, orc_exec_fn exec, void* user);
void orc_engine_free(orc_engine* e);
void orc_push(orc_engine* e, int stage, const void* item);   /* insertIntoQueue / enqueue<S>() */
void orc_record(orc_engine* e, int stage, uint64_t id);        /* trace hook, called by exec fns */
int  orc_run(orc_engine* e);                                   /* fixpoint; returns 0 or error   */

/* ---------------- toy pipeline, Fig. 9 (toy.c) ---------------- */
typedef struct orc_stats { uint64_t deq[ORC_MAX_STAGES], enq[ORC_MAX_STAGES]; } orc_stats;
int orc_toy_definition(const int32_t* in, size_t n, int32_t threshold, int32_t* out, uint64_t* s1_passes);
int orc_toy_pipeline(const int32_t* in, size_t n, int32_t threshold, int32_t* out, size_t* n_out,
                     orc_stats* st);
/* ldpc.c: LDPC decoder, Fig. 17; H as data, edges in check-major order */
typedef struct orc_ldpc {
  int32_t N, M, dv, dc, n_frames, n_iter;
  float alpha;            /* min-sum normalisation                               */
  int32_t nc_chk, nc_var;   /* pipeline items: check chunks, variable chunks (R-L6) */
  int32_t pad;
  const int32_t* check_vars; /* [M*dc] variable node of each edge (check-major)  */
  const int32_t* var_edges;  /* [N*dv] edges of each variable node, ascending    */
  const float* llr;          /* [n_frames*N] channel LLRs                        */
} orc_ldpc;
int orc_ldpc_definition(const orc_ldpc* d, float* post, int32_t* errors);
int orc_ldpc_pipeline(const orc_ldpc* d, float* post, int32_t* errors, orc_stats* st);
/* qbench.c: queue microbenchmark */
int orc_qbench_pipeline(const void* seeds, size_t n, size_t item_bytes, uint32_t fanout, uint64_t* leaves,
                        uint64_t* idsum, uint64_t* bad, orc_stats* st);

/* ---------------- Collatz queue stress (collatz.c) ---------------- */
typedef struct orc_collatz_item { uint32_t id, steps; uint64_t v; } orc_collatz_item;
int orc_collatz_definition(const orc_collatz_item* in, size_t n, uint32_t* steps_out);
int orc_collatz_pipeline(const orc_collatz_item* in, size_t n, uint32_t max_steps, uint32_t* steps_out,
                         uint32_t* seen, orc_stats* st);

/* ---------------- Reyes (reyes.c) ---------------- */
typedef struct orc_patch {
  float cp[16][4]; /* P[a][b] at cp[4a+b], a = u index, b = v index; (x,y,z,1) */
  uint32_t id;     /* frame << 12 | patch                                      */
  uint32_t path;   /* bit d: 0 = left, 1 = right child taken at depth d        */
  uint32_t dirs;   /* bit d: split direction at depth d (0 = u, 1 = v)         */
  uint32_t depth;
} orc_patch;

typedef struct orc_reyes_scene {
  int32_t W, H, n_frames, patches_per_frame, max_depth, pad0;
  float t_dice, near_w;
  const float* M;      /* [n_frames][16] row-major                 */
  const float* albedo; /* [patches_per_frame][4]                   */
  float L[4];
} orc_reyes_scene;

typedef struct orc_reyes_out {
  uint64_t* key;   /* [n_frames*H*W], UINT64_MAX = uncovered                     */
  float* s;        /* [n_frames*H*W] shade factor of the winning micropolygon    */
  float* colour;   /* [n_frames*H*W*4] resolved colour (rgb, alpha = coverage)   */
  /* counts */
  uint64_t n_bound, n_split, n_dice, n_shade, n_culled;
  uint64_t depth_hist[16];        /* leaves (diced) per depth                     */
  uint64_t culled_depth_hist[16]; /* culled nodes per depth                       */
  /* optional: leaf node ids (id << 12 | depth << 8 | path) and their grids */
  uint64_t* leaf_ids; size_t leaf_cap, n_leaves;
  float* leaf_grids;  /* [leaf_cap][6][81]: x, y, z, sx, sy, zs (SoA per leaf)        */
  /* optional per-stage trace (pipeline oracle only) */
  orc_trace_rec* trace; size_t trace_cap, trace_n;
  /* micropolygons whose Q8 bounding box (clamped to the screen) holds a pixel centre:
   * the ones Shade has to rasterise (the GPU reports the same count, vp_run_stats.work_units) */
  uint64_t n_mp_covering;
} orc_reyes_out;

enum { ORC_REYES_CULL = 0, ORC_REYES_SPLIT = 1, ORC_REYES_DICE = 2 };

int orc_reyes_definition(const orc_reyes_scene* sc, const orc_patch* seeds, size_t n, orc_reyes_out* out);
int orc_reyes_pipeline(const orc_reyes_scene* sc, const orc_patch* seeds, size_t n, orc_reyes_out* out);
/* exposed pieces, so tests can pin them individually against independent math */
int  orc_reyes_bound(const orc_reyes_scene* sc, const orc_patch* p, int* split_dir);
void orc_reyes_split(const orc_patch* p, int dir, orc_patch* left, orc_patch* right);
void orc_reyes_dice(const orc_reyes_scene* sc, const orc_patch* p, float grid[6][81]);
void orc_reyes_project(const float M[16], const float p[4], float c[4]);
float orc_reyes_shade_factor(const float n[3], const float L[4]);

/* ---------------- Rasterization (raster.c) ---------------- */
typedef struct orc_raster_scene {
  int32_t W, H;
  int64_t n_tris;
  const float* M;   /* [16] row-major                                   */
  const float* pos; /* [n_tris][3][4] (x_px, y_px, z, 1)                 */
  const float* col; /* [n_tris][3][4] (r, g, b, 0)                       */
  int32_t near_clip; /* 1: clip against z = 0, keys carry sub-ids 2 tri + j (R-S9) */
} orc_raster_scene;

typedef struct orc_raster_out {
  uint64_t* key;   /* [H*W] min (zkey(z) << 32 | tri), UINT64_MAX if empty */
  float* colour;   /* [H*W][4]                                          */
  uint64_t n_vertex, n_clip, n_raster, n_fragment, n_frag_pixels;
  orc_trace_rec* trace; size_t trace_cap, trace_n;
} orc_raster_out;

/* ---------------- Image pyramid (pyramid.c) ---------------- */
typedef struct orc_pyr_scene {
  int32_t S;          /* image side, a power of two >= 64 */
  int32_t n_img;
  const uint8_t* rgb; /* [n_img][S][S][3] */
} orc_pyr_scene;

typedef struct orc_pyr_out {
  uint8_t* gray;  /* [n_img][S*S] level-0 grayscale (before equalisation) */
  uint32_t* hist; /* [n_img][256] */
  uint8_t* lut;   /* [n_img][256] */
  uint8_t* pyr;   /* [n_img][sum_l (S>>l)^2] levels concatenated, level 0 equalised */
  uint64_t n_gray, n_cdf, n_map, n_resize;
  orc_trace_rec* trace; size_t trace_cap, trace_n;
} orc_pyr_out;

int orc_pyr_levels(int S);
size_t orc_pyr_level_offset(int S, int l);
void orc_histeq_lut(const uint32_t hist[256], uint64_t N, uint8_t lut[256]);
int orc_pyr_definition(const orc_pyr_scene* sc, orc_pyr_out* out);
int orc_pyr_pipeline(const orc_pyr_scene* sc, orc_pyr_out* out);

/* ---------------- CFD (cfd.c) ---------------- */
typedef struct orc_cfd_scene {
  int32_t G;              /* grid side (cells)                                     */
  int32_t T;              /* cells per tile item (divides G)                        */
  int32_t n_outer;        /* outer iterations (each: Copy, StepFactor, 3 x RK)      */
  int32_t pad;
  const float* vars0;     /* [5][G*G] initial conserved variables (SoA)              */
  const float* area;      /* [G*G]                                                  */
  const int32_t* nb;      /* [4][G*G] neighbour cell or -1 (wall) / -2 (far field)  */
  const float* normals;   /* [4][3][G*G]                                            */
  float ff[5];            /* far-field conserved state                               */
} orc_cfd_scene;

typedef struct orc_cfd_out {
  float* vars;            /* [5][G*G] final state                                    */
  uint64_t n_copy, n_step, n_flux, n_time;
  orc_trace_rec* trace; size_t trace_cap, trace_n;
} orc_cfd_out;

int orc_cfd_definition(const orc_cfd_scene* sc, orc_cfd_out* out);
int orc_cfd_pipeline(const orc_cfd_scene* sc, orc_cfd_out* out);

/* ---------------- LBP face detection (facedet.c) ---------------- */
typedef struct orc_fd_scene {
  int32_t W, H, n_frames, n_stages;
  const uint8_t* rgb;      /* [n_frames][H][W][3]                                   */
  int32_t n_weak[16];      /* weak classifiers per cascade stage                     */
  int32_t thr[16];         /* stage thresholds                                       */
  const int32_t* weak;     /* [sum n_weak][12]: cx, cy, mask[8], in, out             */
} orc_fd_scene;

typedef struct orc_fd_out {
  uint8_t* levels;         /* [n_frames][sum_l W_l*H_l] equalised pyramid             */
  uint8_t* lbp;            /* [n_frames][sum_l W_l*H_l] LBP codes                    */
  uint32_t* hist;          /* [n_frames][256]                                        */
  uint8_t* lut;            /* [n_frames][256]                                        */
  uint32_t* det;           /* [det_cap][4] frame, level, x, y                         */
  size_t det_cap, n_det;
  uint64_t survivors[16];  /* windows passing cascade stage k                         */
  uint64_t windows;        /* windows evaluated                                       */
  uint64_t deq[8];
  orc_trace_rec* trace; size_t trace_cap, trace_n;
} orc_fd_out;

int orc_fd_levels(int W, int H, int* Ws, int* Hs);
int orc_fd_definition(const orc_fd_scene* sc, orc_fd_out* out);
int orc_fd_pipeline(const orc_fd_scene* sc, orc_fd_out* out);

int orc_raster_definition(const orc_raster_scene* sc, orc_raster_out* out);
int orc_raster_pipeline(const orc_raster_scene* sc, orc_raster_out* out);
void orc_raster_vertex(const orc_raster_scene* sc, uint32_t tri, float clip[3][4]);

#endif

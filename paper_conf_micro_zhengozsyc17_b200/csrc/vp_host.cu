// vp_host.cu — the C ABI of libvp.so (include/vp.h): pipeline assembly, the
// high-level control of PAPER.md §5 (L27: "puts stages into different kernels and do
// SM assignment for them ... we put each kernel into a separate CUDA stream"), the
// KBK host loop (L13 Fig. 3b), the profiling component and the offline auto-tuner
// (L41–L45, Fig. 10).
#include <cuda_runtime.h>
#include <stdarg.h>
#include <stdio.h>
#include <string.h>

#include <algorithm>
#include <chrono>
#include <string>
#include <thread>
#include <vector>

#include "../../include/vp.h"
#include "vp_family.cuh"

using namespace vp;

namespace {

const FamilyOps* all_families[] = {nullptr, nullptr, nullptr, nullptr, nullptr, nullptr, nullptr, nullptr, nullptr, nullptr, nullptr, nullptr, nullptr};
void init_families() {
  if (!all_families[0]) {
    all_families[8] = family_ldpc();
    all_families[7] = family_qbench4();
    all_families[9] = family_qbench16();
    all_families[10] = family_qbench272();
    all_families[11] = family_qbench4_cs();
    all_families[12] = family_qbench16_cs();
    all_families[5] = family_cfd();
    all_families[6] = family_facedet();
    all_families[0] = family_toy();
    all_families[1] = family_collatz();
    all_families[2] = family_reyes();
    all_families[3] = family_raster();
    all_families[4] = family_pyramid();
  }
}
const FamilyOps* family_of_kind(int kind, int* pos) {
  init_families();
  for (const FamilyOps* f : all_families)
    for (int s = 0; s < f->S; ++s)
      if (f->kinds[s] == kind) {
        *pos = s;
        return f;
      }
  return nullptr;
}

// ---------------------------------------------------------------- device helpers
__global__ void k_init_seq(unsigned long long* seq, unsigned long long cap, unsigned long long start) {
  for (unsigned long long i = blockIdx.x * (unsigned long long)blockDim.x + threadIdx.x; i < cap;
       i += (unsigned long long)gridDim.x * blockDim.x) {
    // slot (start + i) & mask is free for ticket start + i
    unsigned long long t = start + i;
    seq[t & (cap - 1)] = t;
  }
}

struct RunInit {
  long long pending;
  unsigned long long watchdog_ns;
  unsigned long long seeds[kMaxStages];
  long long gpend[kMaxKernels];  // online adaptation: seeds of each group's stages
};

__global__ void k_run_init(Ctrl* c, uint32_t* blk, RunInit ri) {
  int t = threadIdx.x;
  for (int i = t; i < kMaxKernels * kMaxSM; i += blockDim.x) blk[i] = 0;
  if (t < kMaxStages) {
    c->seed_head[t].v = 0;
    c->deq[t] = 0;
    c->enq[t] = ri.seeds[t];
    c->max_depth[t] = 0;
    c->exec_ns[t] = 0;
    c->flush_ns[t] = 0;
  }
  if (t < kMaxKernels) {
    c->idle_ns[t] = 0;
    c->rounds[t] = 0;
  }
  if (t < kMaxStages) {
    c->units[t] = 0;
    c->stolen[t] = 0;
  }
  if (t < kMaxKernels) {
    c->arrivals[t].v = 0;
    c->admitted[t].v = 0;
    c->gpend[t].v = (unsigned long long)ri.gpend[t];
    c->retired[t] = 0;
    c->exits[t] = 0;
  }
  if (t < kMaxStages) c->wave_n[t] = 0;
  if (t == 0) {
    c->graph_iters = 0;
    c->pending.v = (unsigned long long)ri.pending;
    c->abort.v = 0;
    c->trace_n.v = 0;
    c->fallback_admits = 0;
    c->deadline.v = globaltimer() + ri.watchdog_ns;
  }
}

__global__ void k_set_abort(Ctrl* c, unsigned long long why) { atomicCAS(&c->abort.v, 0ull, why); }

// Wave sizing shared by the host-driven and the device-driven KBK loops: the largest wave
// of stage s whose children are guaranteed ring space while no other stage runs.
//  * target t != s: n * f <= cap_t - count_t.
//  * t == s (recursion): every claim takes a ring item while ring items remain, and a
//    block releases a claimed slot before it publishes that item's children, so the
//    ring holds at most count_s + f*n - (ring items claimed) slots: with n_r = min(n,
//    count_s) ring items claimed, count_s + f*n - n_r <= cap_s.
// Zero means "not now" (a downstream wave has to drain a target first).
__host__ __device__ inline long long wave_size(int s, long long ring_s, long long seeds_left, const long long* count,
                                               const long long* cap, const int* fan, int S) {
  long long n = ring_s + seeds_left;
  for (int t = 0; t < S; ++t) {
    const long long f = fan[t];
    if (f <= 0) continue;
    const long long freec = cap[t] - count[t];
    if (freec <= 0) return 0;
    if (t != s) {
      n = n < freec / f ? n : freec / f;
    } else if (f == 1) {
      // children replace claimed ring items one for one; only seed claims need space
      const long long m = ring_s + freec;
      n = n < m ? n : m;
    } else {
      // n <= ring_s: (f-1)*n <= free;  beyond ring_s every extra (seed) item needs f slots
      long long a = freec / (f - 1);
      if (a < ring_s) {
        n = n < a ? n : a;
      } else {
        const long long extra = (freec - (f - 1) * ring_s) / f;
        n = n < ring_s + extra ? n : ring_s + extra;
      }
    }
  }
  return n > 0 ? n : 0;
}

// Device-driven KBK (VP_KBK_GRAPH): the host loop's control logic (read the counts,
// size the next wave) moved into a one-thread planner kernel, and the loop itself into a
// CUDA-graph while node.  Same wave kernels, same wave sizing rule, no host round trip.
struct WavePlan {
  long long n_seeds;            // seeds of this stage
  long long cap[kMaxStages];    // ring slots per stage
  int fan[kMaxStages];          // fan-out of this stage to each stage
  int S;
};
__global__ void k_wave_plan(Ctrl* c, int s, WavePlan wp) {
  long long count[kMaxStages];
  for (int t = 0; t < kMaxStages; ++t) count[t] = t < wp.S ? (long long)c->count[t].v : 0;
  long long left = wp.n_seeds - (long long)c->seed_head[s].v;
  long long n = wave_size(s, count[s], left > 0 ? left : 0, count, wp.cap, wp.fan, wp.S);
  if (c->abort.v != 0) n = 0;
  c->wave_n[s] = n;
}
__global__ void k_wave_cond(Ctrl* c, cudaGraphConditionalHandle h) {
  bool more = (long long)c->pending.v > 0 && c->abort.v == 0;
  if (more && globaltimer() > c->deadline.v) {  // the wave kernels' watchdog, also for empty waves
    atomicCAS(&c->abort.v, 0ull, (unsigned long long)ABORT_TIMEOUT);
    more = false;
  }
  c->graph_iters++;
  cudaGraphSetConditional(h, more ? 1u : 0u);
}

__global__ void k_reset_queues(Ctrl* c) {
  int t = threadIdx.x;
  if (t < kMaxStages) {
    c->tail[t].v = 0;
    c->head[t].v = 0;
    c->count[t].v = 0;
  }
}

// ---------------------------------------------------------------- pipeline object
struct StageRec {
  vp_stage_desc d;
  std::string name;
  int cap_log2 = 0;
  uint8_t* slots = nullptr;
  unsigned long long* seq = nullptr;
  uint8_t* seeds = nullptr;
  size_t seed_cap = 0;  // items
  size_t n_seeds = 0;
};

struct KernelPlan {
  int lo, hi;
  bool rtc;
  int quota;
  uint32_t mask[kMaskWords];
  int grid;
  bool coop;
  int kslot;
  // online adaptation
  int group = -1;        // = kslot of the group's primary kernel
  bool can_retire = false;
  uint32_t feeders = 0;  // groups emitting into this kernel's stages
  int refill = -1;       // kernel whose group gets this kernel's SMs when it retires (if no
                         // candidate has stalled work at that moment)
  uint32_t refill_cands = 0;  // persistent groups downstream of this one (refill candidates)
};

struct Plan {
  int model = -1;
  std::vector<KernelPlan> kernels;     // persistent kernels
  std::vector<int> kbk_stages;         // stages driven by the host wave loop
  bool wave_rtc = false;               // standalone RTC: waves of the [0,S-1] RTC kernel
  bool kbk_graph = false;              // KBK waves driven on the device by a CUDA-graph while loop
  bool online = false;                 // online adaptation (VP_FLAG_ONLINE): retire + refill
  int8_t stage_group[kMaxStages] = {};
  int batch[kMaxStages] = {};
  int cap_log2[kMaxStages] = {};       // effective ring size this plan runs with
  vp_config cfg{};
};

}  // namespace

struct vp_pipeline_s {
  int device = 0;
  int num_sms = 0;
  vp_pipeline_desc desc{};
  const FamilyOps* fam = nullptr;
  std::vector<uint8_t> params;
  std::vector<StageRec> st;
  bool queues_ready = false;
  bool configured = false;
  bool dirty_queues = false;  // after an aborted run: reset rings before the next one
  int run_cap_log2[kMaxStages] = {};  // ring size the seq words were initialised for
  Plan plan;
  Ctrl* ctrl = nullptr;
  uint32_t* blk = nullptr;
  TraceRec* trace = nullptr;
  Ctrl* h_ctrl = nullptr;     // pinned readback
  uint32_t* h_blk = nullptr;
  volatile uint32_t* h_arrive = nullptr;  // mapped pinned: per-kernel dispatch-complete flags
  uint32_t* d_arrive = nullptr;
  volatile uint32_t* h_retire = nullptr;  // mapped pinned: per-kernel "retired, SMs free" flags
  uint32_t* d_retire = nullptr;
  volatile long long* h_gpend = nullptr;  // mapped pinned: group alive counts at each retirement
  long long* d_gpend = nullptr;
  uint32_t epoch = 0;
  cudaStream_t streams[kMaxKernels] = {};
  cudaEvent_t ev_fork = nullptr, ev_start = nullptr, ev_end = nullptr, ev_join[kMaxKernels] = {};
  cudaEvent_t ev_kbeg[kMaxKernels] = {};
  std::string err;
  int kernel_occ_cache[kMaxStages][kMaxStages][2] = {};
  double timeout_ms = 30000;
  // device-driven KBK: instantiated graph and the launch arguments it was captured with
  int refill_lo[kMaxKernels] = {}, refill_hi[kMaxKernels] = {}, refill_quota[kMaxKernels] = {};
  int refill_pick[kMaxKernels] = {};  // kernel whose group each retired kernel's SMs went to
  bool launched[kMaxKernels] = {};  // planned kernels launched by the last vp_run
  // host-driven KBK: per-wave event pairs (pooled) and the stage of each wave of the last run
  std::vector<cudaEvent_t> wave_ev;
  std::vector<int> wave_stage;
  void* seq_arena = nullptr;  // every ring's sequence words (one L2 persisting window)
  size_t seq_arena_bytes = 0;
  bool l2_window_set = false;
  cudaGraph_t kg_graph = nullptr;
  cudaGraphExec_t kg_exec = nullptr;
  std::vector<uint8_t> kg_key;
};

namespace {

vp_status fail(vp_pipeline_s* p, vp_status s, const char* fmt, ...) {
  if (p) {
    char buf[1024];
    va_list ap;
    va_start(ap, fmt);
    vsnprintf(buf, sizeof(buf), fmt, ap);
    va_end(ap);
    p->err = buf;
  }
  return s;
}
#define CUDA_TRY(p, x)                                                                        \
  do {                                                                                        \
    cudaError_t e_ = (x);                                                                     \
    if (e_ != cudaSuccess) {                                                                  \
      return fail((p), e_ == cudaErrorMemoryAllocation ? VP_ERR_OOM : VP_ERR_CUDA, "%s: %s (%s:%d)", #x, \
                  cudaGetErrorString(e_), __FILE__, __LINE__);                                \
    }                                                                                         \
  } while (0)

struct DeviceGuard {
  int prev = -1;
  explicit DeviceGuard(int d) {
    cudaGetDevice(&prev);
    if (prev != d) cudaSetDevice(d);
  }
  ~DeviceGuard() {
    int cur;
    cudaGetDevice(&cur);
    if (prev >= 0 && cur != prev) cudaSetDevice(prev);
  }
};

int occupancy(vp_pipeline_s* p, int lo, int hi, bool rtc) {
  int& c = p->kernel_occ_cache[lo][hi][rtc ? 1 : 0];
  if (c) return c;
  const void* fn = p->fam->kernel(lo, hi, rtc);
  if (!fn) return 0;
  size_t sm = p->fam->smem(lo, hi, rtc);
  cudaFuncSetAttribute(fn, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)sm);
  // One shared-memory carveout for every kernel: an SM configured for a small carveout
  // cannot take a block of a kernel that needs a larger one until it drains, which would
  // stop co-resident persistent groups (coarse/fine/hybrid) from ever starting.
  cudaFuncSetAttribute(fn, cudaFuncAttributePreferredSharedMemoryCarveout, (int)cudaSharedmemCarveoutMaxShared);
  int occ = 0;
  if (cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, fn, p->fam->block_threads(lo, hi, rtc), sm) != cudaSuccess) occ = 0;
  c = occ;
  return occ;
}

void mask_all(uint32_t* m, int nsm) {
  memset(m, 0, sizeof(uint32_t) * kMaskWords);
  for (int i = 0; i < nsm; ++i) m[i >> 5] |= 1u << (i & 31);
}
void mask_range(uint32_t* m, int a, int b) {
  memset(m, 0, sizeof(uint32_t) * kMaskWords);
  for (int i = a; i < b; ++i) m[i >> 5] |= 1u << (i & 31);
}
int mask_count(const uint32_t* m, int nsm) {
  int c = 0;
  for (int i = 0; i < nsm; ++i) c += (m[i >> 5] >> (i & 31)) & 1u;
  return c;
}

vp_status ensure_queues(vp_pipeline_s* p) {
  if (p->queues_ready) return VP_OK;
  // All sequence-word arrays live in one arena, so one L2 access-policy window can pin
  // them (VP_FLAG_L2_PERSIST); each array starts on a 256-B boundary.
  size_t seq_bytes = 0;
  for (size_t s = 0; s < p->st.size(); ++s) seq_bytes += ((1ull << p->st[s].cap_log2) * 8 + 255) / 256 * 256;
  CUDA_TRY(p, cudaMalloc(&p->seq_arena, seq_bytes));
  p->seq_arena_bytes = seq_bytes;
  size_t off = 0;
  for (size_t s = 0; s < p->st.size(); ++s) {
    StageRec& r = p->st[s];
    size_t cap = 1ull << r.cap_log2;
    CUDA_TRY(p, cudaMalloc(&r.slots, cap * (size_t)p->fam->stride((int)s)));
    r.seq = (unsigned long long*)((uint8_t*)p->seq_arena + off);
    off += (cap * 8 + 255) / 256 * 256;
    k_init_seq<<<256, 256>>>(r.seq, cap, 0);
    p->run_cap_log2[s] = r.cap_log2;
    CUDA_TRY(p, cudaGetLastError());
  }
  CUDA_TRY(p, cudaDeviceSynchronize());
  p->queues_ready = true;
  return VP_OK;
}

vp_status reset_queues(vp_pipeline_s* p, cudaStream_t st) {
  k_reset_queues<<<1, 32, 0, st>>>(p->ctrl);
  for (size_t s = 0; s < p->st.size(); ++s) {
    int lg = p->plan.cap_log2[s] ? p->plan.cap_log2[s] : p->st[s].cap_log2;
    p->run_cap_log2[s] = lg;
    k_init_seq<<<256, 256, 0, st>>>(p->st[s].seq, 1ull << lg, 0);
  }
  CUDA_TRY(p, cudaGetLastError());
  p->dirty_queues = false;
  return VP_OK;
}

Common make_common(vp_pipeline_s* p) {
  Common c;
  memset(&c, 0, sizeof(c));
  for (size_t s = 0; s < p->st.size(); ++s) {
    const StageRec& r = p->st[s];
    c.q[s].slots = r.slots;
    c.q[s].seq = r.seq;
    c.q[s].seeds = r.seeds;
    c.q[s].n_seeds = (long long)r.n_seeds;
    c.q[s].cap_log2 = (uint32_t)(p->plan.cap_log2[s] ? p->plan.cap_log2[s] : r.cap_log2);
    c.q[s].stride = (uint32_t)p->fam->stride((int)s);
  }
  c.ctrl = p->ctrl;
  c.blk = p->blk;
  c.trace = p->trace;
  c.trace_cap = (p->desc.flags & VP_FLAG_TRACE) ? (unsigned long long)p->desc.trace_capacity : 0ull;
  c.flags = ((p->desc.flags & VP_FLAG_TRACE) ? FLAG_TRACE : 0u) | ((p->desc.flags & VP_FLAG_QUEUE_DEPTH) ? FLAG_DEPTH : 0u) |
            ((p->desc.flags & VP_FLAG_TIMERS) ? FLAG_TIMERS : 0u) | ((p->desc.flags & VP_FLAG_CLUSTER_STEAL) ? FLAG_STEAL : 0u);
  c.n_stages = (int)p->st.size();
  c.host_arrive = p->d_arrive;
  c.host_retire = p->d_retire;
  c.host_gpend = p->d_gpend;
  c.epoch = p->epoch;
  for (int s = 0; s < kMaxStages; ++s) c.stage_group[s] = p->plan.online ? p->plan.stage_group[s] : (int8_t)-1;
  return c;
}

// Per-block SM resources of a kernel (register allocation per warp in units of 256,
// static + dynamic + 1 KB reserved shared memory).
struct KRes {
  int regs, smem, threads;
};
KRes kernel_res(vp_pipeline_s* p, int lo, int hi, bool rtc) {
  const int nt = p->fam->block_threads(lo, hi, rtc);
  KRes r{0, 0, nt};
  cudaFuncAttributes at;
  if (cudaFuncGetAttributes(&at, p->fam->kernel(lo, hi, rtc)) != cudaSuccess) return KRes{1 << 30, 1 << 30, nt};
  int per_warp = ((at.numRegs * 32 + 255) / 256) * 256;
  r.regs = per_warp * (nt / 32);
  r.smem = (int)(at.sharedSizeBytes + p->fam->smem(lo, hi, rtc)) + 1024;
  return r;
}
bool fits_sm(vp_pipeline_s* p, const KRes* res, const int* q, int n) {
  cudaDeviceProp prop;
  cudaGetDeviceProperties(&prop, p->device);
  long long regs = 0, smem = 0, thr = 0, blocks = 0;
  for (int i = 0; i < n; ++i) {
    regs += (long long)q[i] * res[i].regs;
    smem += (long long)q[i] * res[i].smem;
    thr += (long long)q[i] * res[i].threads;
    blocks += q[i];
  }
  return regs <= prop.regsPerMultiprocessor && smem <= (long long)prop.sharedMemPerMultiprocessor &&
         thr <= prop.maxThreadsPerMultiProcessor && blocks <= prop.maxBlocksPerMultiProcessor;
}
// Block mapping of a fine group [lo,hi] (Fig. 5; Block Mapping Controller, L27): every
// stage kernel gets the same block quota on each of its SMs (L45 pruning rule).  If all
// stages cannot co-reside on one SM, SM j of the group hosts the cyclic window of m
// stages {(j + i) mod n : i < m} for the largest m whose every window fits.
// Requested quotas are checked; missing ones are filled greedily (round-robin while
// every window still fits).
vp_status fine_quotas(vp_pipeline_s* p, int lo, int hi, const int* req, const uint32_t* group_mask, int* q,
                      uint32_t (*masks)[kMaskWords]) {
  const int n = hi - lo + 1;
  KRes res[kMaxStages];
  int qq[kMaxStages];
  bool fixed[kMaxStages];
  for (int i = 0; i < n; ++i) {
    res[i] = kernel_res(p, lo + i, lo + i, false);
    fixed[i] = req && req[lo + i] > 0;
    qq[i] = fixed[i] ? req[lo + i] : 1;
  }
  auto windows_fit = [&](int m) {
    for (int j = 0; j < n; ++j) {
      KRes wr[kMaxStages];
      int wq[kMaxStages];
      for (int i = 0; i < m; ++i) {
        wr[i] = res[(j + i) % n];
        wq[i] = qq[(j + i) % n];
      }
      if (!fits_sm(p, wr, wq, m)) return false;
      if (m == n) break;
    }
    return true;
  };
  int m = n;
  while (m > 0 && !windows_fit(m)) --m;
  if (m == 0)
    return fail(p, VP_ERR_INVALID, "fine group [%d,%d]: block quotas do not fit one SM (registers/smem/threads)", lo, hi);
  for (bool grew = true; grew;) {
    grew = false;
    for (int i = 0; i < n; ++i) {
      if (fixed[i]) continue;
      qq[i]++;
      if (windows_fit(m)) grew = true;
      else qq[i]--;
    }
  }
  for (int i = 0; i < n; ++i) {
    q[lo + i] = qq[i];
    memset(masks[lo + i], 0, sizeof(uint32_t) * kMaskWords);
  }
  int j = 0;
  for (int sm = 0; sm < kMaxSM; ++sm) {
    if (!((group_mask[sm >> 5] >> (sm & 31)) & 1u)) continue;
    for (int i = 0; i < m; ++i) {
      int st = lo + (j + i) % n;
      masks[st][sm >> 5] |= 1u << (sm & 31);
    }
    ++j;
  }
  return VP_OK;
}

vp_status build_plan(vp_pipeline_s* p, int model, const vp_sm_binding* b, int batch, Plan& out) {
  const int S = (int)p->st.size();
  const int N = p->num_sms;
  Plan pl;
  pl.model = model;
  for (int s = 0; s < S; ++s) {
    int bs = p->fam->default_batch(s);
    if (b && b->batch[s] > 0) bs = b->batch[s];
    if (batch > 0) bs = batch;
    if (bs > p->fam->max_batch(s)) bs = p->fam->max_batch(s);
    if (bs < 1) return fail(p, VP_ERR_INVALID, "batch for stage %d must be >= 1", s);
    pl.batch[s] = bs;
  }
  auto add_kernel = [&](int lo, int hi, bool rtc, int quota, const uint32_t* mask, bool coop) -> vp_status {
    int occ = occupancy(p, lo, hi, rtc);
    if (occ <= 0) return fail(p, VP_ERR_UNSUPPORTED, "kernel [%d,%d]%s cannot be resident (occupancy 0)", lo, hi, rtc ? " RTC" : "");
    if (quota > occ) return fail(p, VP_ERR_INVALID, "infeasible block quota %d > %d resident blocks/SM for stages [%d,%d]", quota, occ, lo, hi);
    KernelPlan k;
    k.lo = lo;
    k.hi = hi;
    k.rtc = rtc;
    k.quota = quota;
    memcpy(k.mask, mask, sizeof(k.mask));
    k.coop = coop;
    int per = quota > 0 ? quota : occ;
    // filling-retreating (L27): enough blocks to fill every SM.  A kernel with a block
    // quota (fine groups) launches exactly quota x (its SMs) blocks: its quotas and its
    // co-resident kernels' fill the SMs, so surplus blocks would have no SM to retreat
    // through and would stall the dispatch of every later grid (seen with 4 fine LDPC
    // stage kernels at 1 block/SM each).
    k.grid = coop ? per * N : (quota > 0 ? quota * std::max(1, mask_count(mask, N)) : occ * N);
    k.kslot = (int)pl.kernels.size();
    if (k.kslot >= kMaxKernels) return fail(p, VP_ERR_INVALID, "too many kernels");
    pl.kernels.push_back(k);
    return VP_OK;
  };
  uint32_t all[kMaskWords];
  mask_all(all, N);
  vp_status rc = VP_OK;
  switch (model) {
    case VP_RTC:
      if (!p->fam->rtc_legal(0, S - 1))
        return fail(p, VP_ERR_UNSUPPORTED, "RTC needs a linear pipeline without recursion, loops or global sync (L11)");
      pl.wave_rtc = true;
      break;
    case VP_KBK:
    case VP_KBK_GRAPH:
      for (int s = 0; s < S; ++s) pl.kbk_stages.push_back(s);
      pl.kbk_graph = model == VP_KBK_GRAPH;
      break;
    case VP_MEGAKERNEL: {
      int q = (b && b->blocks_per_sm[0] > 0) ? b->blocks_per_sm[0] : 0;
      rc = add_kernel(0, S - 1, false, q, all, true);
      break;
    }
    case VP_COARSE: {
      // each stage its own persistent kernel on exclusive SMs (Fig. 4, L21)
      for (int s = 0; s < S && rc == VP_OK; ++s) {
        uint32_t m[kMaskWords];
        if (b) memcpy(m, b->group_sm_mask[s], sizeof(m));
        else mask_range(m, s * N / S, (s + 1) * N / S);
        int q = (b && b->blocks_per_sm[s] > 0) ? b->blocks_per_sm[s] : 0;
        rc = add_kernel(s, s, false, q, m, false);
      }
      break;
    }
    case VP_FINE: {
      // each stage its own persistent kernel; SMs shared, blocks per (stage, SM) capped (Fig. 5)
      int q[kMaxStages];
      uint32_t sm_of[kMaxStages][kMaskWords];
      uint32_t m[kMaskWords];
      if (b && b->num_groups == 1) memcpy(m, b->group_sm_mask[0], sizeof(m));
      else memcpy(m, all, sizeof(m));
      rc = fine_quotas(p, 0, S - 1, b ? b->blocks_per_sm : nullptr, m, q, sm_of);
      for (int s = 0; s < S && rc == VP_OK; ++s) rc = add_kernel(s, s, false, q[s], sm_of[s], false);
      break;
    }
    case VP_HYBRID: {
      if (!b) return fail(p, VP_ERR_INVALID, "VP_HYBRID needs a vp_sm_binding");
      int G = b->num_groups;
      if (G < 1 || G > S) return fail(p, VP_ERR_INVALID, "num_groups must be in [1, %d]", S);
      int lo[kMaxStages], hi[kMaxStages];
      for (int g = 0; g < G; ++g) lo[g] = S, hi[g] = -1;
      for (int s = 0; s < S; ++s) {
        int g = b->group_of_stage[s];
        if (g < 0 || g >= G) return fail(p, VP_ERR_INVALID, "group_of_stage[%d] out of range", s);
        if (s > 0 && g != b->group_of_stage[s - 1] && g != b->group_of_stage[s - 1] + 1)
          return fail(p, VP_ERR_INVALID, "groups must be contiguous stage ranges in order (L45)");
        if (s == 0 && g != 0) return fail(p, VP_ERR_INVALID, "stage 0 must be in group 0");
        lo[g] = std::min(lo[g], s);
        hi[g] = std::max(hi[g], s);
      }
      // Groups normally own disjoint SMs (coarse pipelining between groups, L27).  Groups may
      // share SMs -- a fine pipeline between groups (Fig. 5's per-SM block quotas, applied to
      // group kernels) -- when every group on a shared SM is a MEGA or RTC group with an
      // explicit block quota and the quotas of all groups on that SM fit it together.
      for (int g = 0; g < G; ++g) {
        if (hi[g] < 0) return fail(p, VP_ERR_INVALID, "group %d is empty", g);
        if (mask_count(b->group_sm_mask[g], N) == 0) return fail(p, VP_ERR_INVALID, "group %d has no SM in its mask", g);
      }
      for (int sm = 0; sm < N; ++sm) {
        int on[kMaxStages], non = 0;
        for (int g = 0; g < G; ++g)
          if ((b->group_sm_mask[g][sm >> 5] >> (sm & 31)) & 1u) on[non++] = g;
        if (non < 2) continue;
        KRes res[kMaxStages];
        int qs[kMaxStages];
        for (int i = 0; i < non; ++i) {
          const int g = on[i], gm = b->group_model[g], q = b->blocks_per_sm[lo[g]];
          if ((gm != VP_GROUP_MEGA && gm != VP_GROUP_RTC) || q <= 0)
            return fail(p, VP_ERR_INVALID, "SM masks of groups overlap (SM %d): only MEGA/RTC groups with explicit "
                                           "blocks_per_sm quotas may share SMs (coarse pipelining between groups, L27)", sm);
          if (gm == VP_GROUP_RTC && !p->fam->rtc_legal(lo[g], hi[g]))
            return fail(p, VP_ERR_UNSUPPORTED, "RTC group [%d,%d] has recursion, a loop or a latch", lo[g], hi[g]);
          res[i] = kernel_res(p, lo[g], hi[g], gm == VP_GROUP_RTC);
          qs[i] = q;
        }
        if (!fits_sm(p, res, qs, non))
          return fail(p, VP_ERR_INVALID, "groups sharing SM %d: their block quotas do not fit one SM together", sm);
      }
      for (int g = 0; g < G && rc == VP_OK; ++g) {
        int gm = b->group_model[g];
        const uint32_t* m = b->group_sm_mask[g];
        if (gm == VP_GROUP_RTC) {
          if (!p->fam->rtc_legal(lo[g], hi[g]))
            return fail(p, VP_ERR_UNSUPPORTED, "RTC group [%d,%d] has recursion, a loop or a latch", lo[g], hi[g]);
          rc = add_kernel(lo[g], hi[g], true, b->blocks_per_sm[lo[g]], m, false);
        } else if (gm == VP_GROUP_MEGA) {
          rc = add_kernel(lo[g], hi[g], false, b->blocks_per_sm[lo[g]], m, false);
        } else if (gm == VP_GROUP_FINE) {
          int q[kMaxStages];
          uint32_t sm_of[kMaxStages][kMaskWords];
          rc = fine_quotas(p, lo[g], hi[g], b->blocks_per_sm, m, q, sm_of);
          for (int s = lo[g]; s <= hi[g] && rc == VP_OK; ++s) rc = add_kernel(s, s, false, q[s], sm_of[s], false);
        } else if (gm == VP_GROUP_KBK) {
          for (int s = lo[g]; s <= hi[g]; ++s) pl.kbk_stages.push_back(s);
        } else {
          return fail(p, VP_ERR_INVALID, "unknown group model %d", gm);
        }
      }
      break;
    }
    default:
      return fail(p, VP_ERR_INVALID, "unknown model %d", model);
  }
  if (rc != VP_OK) return rc;
  // per-kernel batch caps (a stage is fetched by exactly one kernel or wave kind)
  auto clamp_batch = [&](int lo, int hi, bool rtc) {
    for (int s = lo; s <= hi; ++s) pl.batch[s] = std::min(pl.batch[s], p->fam->max_batch_k(lo, hi, rtc, s));
  };
  for (const KernelPlan& k : pl.kernels) clamp_batch(k.lo, k.hi, k.rtc);
  for (int s : pl.kbk_stages) clamp_batch(s, s, false);
  if (pl.wave_rtc) clamp_batch(0, S - 1, true);
  // Effective ring sizes.  Persistent plans drain continuously: a ring needs room for
  // the batches its producers hold (two out buffers per block), so it is sized to that
  // and stays L2-resident (no dirty-line write-back to HBM).  Host-driven waves (KBK,
  // RTC waves) need room for a whole wave: they use the full allocation.
  for (int t = 0; t < S; ++t) {
    int full = p->st[t].cap_log2;
    if (!pl.kbk_stages.empty() || pl.wave_rtc || (p->desc.flags & VP_FLAG_FULL_RINGS)) {
      pl.cap_log2[t] = full;
      continue;
    }
    // The recursive stages of a block-local-recursion kernel hold its stack overflow: a
    // breadth of deep trees (many seeds recursing at once) can need far more than the
    // producers' batches, so they keep the registered capacity.
    bool rec_target = false;
    for (const KernelPlan& k : pl.kernels)
      if (p->fam->local_rec(k.lo, k.hi, k.rtc) && t >= k.lo && t <= k.hi) rec_target = true;
    if (rec_target) {
      pl.cap_log2[t] = full;
      continue;
    }
    long long need = 0;
    for (const KernelPlan& k : pl.kernels) {
      int per = k.quota > 0 ? k.quota : occupancy(p, k.lo, k.hi, k.rtc);
      long long blocks = (long long)per * mask_count(k.mask, N);
      long long mx = 0;
      for (int s = k.lo; s <= k.hi; ++s) mx = std::max(mx, (long long)pl.batch[s] * p->fam->fanout(s, t));
      // block-local recursion publishes up to its out-buffer capacity per batch
      if (p->fam->local_rec(k.lo, k.hi, k.rtc)) mx = std::max(mx, (long long)p->fam->out_cap(k.lo, k.hi, false, t));
      need += 2 * blocks * mx;
    }
    int lg = 12;
    while (lg < full && (1ll << lg) < need) ++lg;
    pl.cap_log2[t] = std::min(lg, full);
  }
  // every producer batch must fit twice into its target ring, or the ring cannot drain
  for (int s = 0; s < S; ++s)
    for (int t = 0; t < S; ++t) {
      int f = p->fam->fanout(s, t);
      if (f > 0 && 2ll * pl.batch[s] * f > (1ll << pl.cap_log2[t]))
        return fail(p, VP_ERR_INVALID, "queue_capacity of stage %d (%lld) < 2 x batch(%d) x fanout(%d) of stage %d", t,
                    1ll << pl.cap_log2[t], pl.batch[s], f, s);
    }
  // Online adaptation (VP_FLAG_ONLINE; "online tuner ... adjusting SM
  // mappings"): each persistent kernel is a group; a group may retire once nothing can
  // reach its stages (all its feeders are persistent groups that retired), and its SMs go
  // to the first persistent group downstream of it.  KBK stages never retire.
  for (int s = 0; s < kMaxStages; ++s) pl.stage_group[s] = -1;
  pl.online = (p->desc.flags & VP_FLAG_ONLINE) && pl.kbk_stages.empty() && !pl.wave_rtc && pl.kernels.size() > 1;
  if (pl.online) {
    for (KernelPlan& k : pl.kernels) {
      k.group = k.kslot;
      for (int s = k.lo; s <= k.hi; ++s) pl.stage_group[s] = (int8_t)k.kslot;
    }
    for (KernelPlan& k : pl.kernels) {
      k.can_retire = !k.coop;
      for (int s = 0; s < S; ++s) {
        if (s >= k.lo && s <= k.hi) continue;
        bool feeds = false;
        for (int t = k.lo; t <= k.hi; ++t) feeds |= p->fam->fanout(s, t) > 0;
        if (feeds) k.feeders |= 1u << pl.stage_group[s];
      }
      int best = -1;
      for (const KernelPlan& j : pl.kernels)
        if (j.lo > k.hi && !j.coop) {
          k.refill_cands |= 1u << j.kslot;
          if (best < 0 || j.lo < pl.kernels[best].lo) best = j.kslot;
        }
      k.refill = best;
    }
  }
  pl.cfg.model = model;
  pl.cfg.has_binding = b ? 1 : 0;
  if (b) pl.cfg.binding = *b;
  pl.cfg.batch = batch;
  out = pl;
  return VP_OK;
}

// ------------------------------------------------------------------ running
vp_status launch_wave(vp_pipeline_s* p, const Common& c, int lo, int hi, bool rtc, int stage, long long n,
                      cudaStream_t st, int kslot) {
  GroupArgs g;
  memset(&g, 0, sizeof(g));
  g.mode = MODE_WAVE;
  g.wave_stage = stage;
  g.wave_n = n;
  g.kslot = kslot;
  for (int s = 0; s < kMaxStages; ++s) g.batch[s] = p->plan.batch[s] ? p->plan.batch[s] : 1;
  // one resident wave of blocks, each taking a contiguous chunk of whole batches so the
  // fetch / execute / publish warps of a block overlap across its batches
  long long batches = (n + g.batch[stage] - 1) / g.batch[stage];
  long long resident = (long long)std::max(1, occupancy(p, lo, hi, rtc)) * p->num_sms;
  long long grid = std::min(batches, resident);
  g.wave_chunk = ((batches + grid - 1) / grid) * g.batch[stage];
  grid = (n + g.wave_chunk - 1) / g.wave_chunk;
  CUDA_TRY(p, p->fam->launch(lo, hi, rtc, c, g, p->params.data(), (int)grid, false, st));
  return VP_OK;
}

struct Avail {
  long long ring[kMaxStages];
  long long seeds_left[kMaxStages];
  long long pending;
  unsigned long long abort;
};

vp_status read_avail(vp_pipeline_s* p, cudaStream_t st, Avail& a) {
  // the counters live on separate 128-B lines: copy the first kMaxStages*4 + 2 lines
  size_t bytes = offsetof(Ctrl, deadline);
  CUDA_TRY(p, cudaMemcpyAsync(p->h_ctrl, p->ctrl, bytes, cudaMemcpyDeviceToHost, st));
  CUDA_TRY(p, cudaStreamSynchronize(st));
  for (size_t s = 0; s < p->st.size(); ++s) {
    a.ring[s] = (long long)p->h_ctrl->count[s].v;
    long long sh = (long long)p->h_ctrl->seed_head[s].v;
    long long left = (long long)p->st[s].n_seeds - sh;
    a.seeds_left[s] = left > 0 ? left : 0;
  }
  a.pending = (long long)p->h_ctrl->pending.v;
  a.abort = p->h_ctrl->abort.v;
  return VP_OK;
}

vp_status host_wave_loop(vp_pipeline_s* p, const Common& c, cudaStream_t st, uint64_t* launches) {
  // KBK (Fig. 3b): "The pipeline logic control is implemented on the CPU side" — read the
  // queue counts back, launch one kernel for one stage over the items present, repeat.
  // Stage choice: most downstream non-empty stage first (bounds live items, like the
  // task scheduler's priority).  A wave is capped so its output fits the target rings.
  const std::vector<int>& ks = p->plan.kbk_stages;
  const int S = (int)p->st.size();
  long long caps[kMaxStages] = {};
  int fans[kMaxStages][kMaxStages] = {};
  for (int t = 0; t < S; ++t) caps[t] = 1ll << p->plan.cap_log2[t];
  for (int s = 0; s < S; ++s)
    for (int t = 0; t < S; ++t) fans[s][t] = p->fam->fanout(s, t);
  auto wave_n = [&](int s, const Avail& a) -> long long {
    return wave_size(s, a.ring[s], a.seeds_left[s], a.ring, caps, fans[s], S);
  };
  const auto t_start = std::chrono::steady_clock::now();
  for (;;) {
    Avail a;
    vp_status rc = read_avail(p, st, a);
    if (rc != VP_OK) return rc;
    if (a.abort) return VP_OK;
    if (a.pending <= 0) return VP_OK;
    if (std::chrono::duration<double, std::milli>(std::chrono::steady_clock::now() - t_start).count() > p->timeout_ms) {
      // host-side watchdog for wave-driven models (timeoutexec): abort the device run
      k_set_abort<<<1, 1, 0, st>>>(p->ctrl, ABORT_TIMEOUT);
      CUDA_TRY(p, cudaStreamSynchronize(st));
      return VP_OK;
    }
    bool launched = false;
    // VP_FLAG_TIMERS: one event pair per wave (from a pool), read back after the run for
    // stage_wave_ms (off by default: the records would slow the KBK baseline down)
    const bool wave_times = (p->desc.flags & VP_FLAG_TIMERS) != 0;
    auto wave_begin = [&](int s) -> vp_status {
      if (!wave_times) return VP_OK;
      const size_t i = p->wave_stage.size();
      while (p->wave_ev.size() < 2 * (i + 1)) {
        cudaEvent_t e;
        CUDA_TRY(p, cudaEventCreate(&e));
        p->wave_ev.push_back(e);
      }
      p->wave_stage.push_back(s);
      CUDA_TRY(p, cudaEventRecord(p->wave_ev[2 * i], st));
      return VP_OK;
    };
    auto wave_end = [&]() -> vp_status {
      if (!wave_times) return VP_OK;
      CUDA_TRY(p, cudaEventRecord(p->wave_ev[2 * (p->wave_stage.size() - 1) + 1], st));
      return VP_OK;
    };
    if (p->plan.wave_rtc) {
      for (int s = 0; s < S && !launched; ++s) {
        long long n = wave_n(s, a);
        if (n > 0) {
          if ((rc = wave_begin(s)) != VP_OK) return rc;
          rc = launch_wave(p, c, 0, S - 1, true, s, n, st, 0);
          if (rc != VP_OK) return rc;
          if ((rc = wave_end()) != VP_OK) return rc;
          launched = true;
        }
      }
    } else {
      for (int i = (int)ks.size() - 1; i >= 0 && !launched; --i) {
        int s = ks[i];
        long long n = wave_n(s, a);
        if (n > 0) {
          if ((rc = wave_begin(s)) != VP_OK) return rc;
          rc = launch_wave(p, c, s, s, false, s, n, st, 0);
          if (rc != VP_OK) return rc;
          if ((rc = wave_end()) != VP_OK) return rc;
          launched = true;
        }
      }
    }
    if (launched) {
      (*launches)++;
    } else {
      // hybrid: the work is in persistent groups right now; poll again shortly
      std::this_thread::sleep_for(std::chrono::microseconds(5));
    }
  }
}

// Device-driven KBK: one CUDA graph whose while node repeats
//   for s = S-1 .. 0 (downstream first, the host loop's priority):
//     k_wave_plan(s)  -> wave size from the live counts, capped like host_wave_loop
//     wave kernel(s)  -> fixed grid of resident blocks; blocks past the wave exit at once
//   k_wave_cond      -> continue while pending > 0 (and no abort / watchdog)
// The graph is captured once per (plan, queue layout, params) and relaunched.
vp_status graph_wave_run(vp_pipeline_s* p, const Common& c0, cudaStream_t st, uint64_t* launches) {
  const int S = (int)p->st.size();
  Common c = c0;
  c.epoch = 0;  // only persistent blocks use it
  std::vector<uint8_t> key(sizeof(Common) + p->params.size() + sizeof(p->plan.batch) + sizeof(p->plan.cap_log2));
  memcpy(key.data(), &c, sizeof(Common));
  memcpy(key.data() + sizeof(Common), p->params.data(), p->params.size());
  memcpy(key.data() + sizeof(Common) + p->params.size(), p->plan.batch, sizeof(p->plan.batch));
  memcpy(key.data() + sizeof(Common) + p->params.size() + sizeof(p->plan.batch), p->plan.cap_log2, sizeof(p->plan.cap_log2));
  if (!p->kg_exec || key != p->kg_key) {
    if (p->kg_exec) cudaGraphExecDestroy(p->kg_exec);
    if (p->kg_graph) cudaGraphDestroy(p->kg_graph);
    p->kg_exec = nullptr;
    p->kg_graph = nullptr;
    cudaGraph_t g;
    CUDA_TRY(p, cudaGraphCreate(&g, 0));
    p->kg_graph = g;
    cudaGraphConditionalHandle h;
    CUDA_TRY(p, cudaGraphConditionalHandleCreate(&h, g, 1u, cudaGraphCondAssignDefault));
    cudaGraphNodeParams np = {};
    np.type = cudaGraphNodeTypeConditional;
    np.conditional.handle = h;
    np.conditional.type = cudaGraphCondTypeWhile;
    np.conditional.size = 1;
    cudaGraphNode_t node;
    CUDA_TRY(p, cudaGraphAddNode(&node, g, nullptr, 0, &np));
    cudaGraph_t body = np.conditional.phGraph_out[0];
    cudaStream_t cs;
    CUDA_TRY(p, cudaStreamCreateWithFlags(&cs, cudaStreamNonBlocking));
    cudaError_t ce = cudaStreamBeginCaptureToGraph(cs, body, nullptr, nullptr, 0, cudaStreamCaptureModeRelaxed);
    if (ce != cudaSuccess) {
      cudaStreamDestroy(cs);
      CUDA_TRY(p, ce);
    }
    const std::vector<int>& ks = p->plan.kbk_stages;
    for (int i = (int)ks.size() - 1; i >= 0 && ce == cudaSuccess; --i) {
      const int s = ks[i];
      WavePlan wp;
      memset(&wp, 0, sizeof(wp));
      wp.n_seeds = (long long)p->st[s].n_seeds;
      wp.S = S;
      for (int t = 0; t < S; ++t) {
        wp.fan[t] = p->fam->fanout(s, t);
        wp.cap[t] = 1ll << p->plan.cap_log2[t];
      }
      k_wave_plan<<<1, 1, 0, cs>>>(p->ctrl, s, wp);
      GroupArgs ga;
      memset(&ga, 0, sizeof(ga));
      ga.mode = MODE_WAVE;
      ga.wave_stage = s;
      ga.wave_n_dev = &p->ctrl->wave_n[s];
      for (int t = 0; t < kMaxStages; ++t) ga.batch[t] = p->plan.batch[t] ? p->plan.batch[t] : 1;
      int grid = std::max(1, occupancy(p, s, s, false)) * p->num_sms;
      ce = p->fam->launch(s, s, false, c, ga, p->params.data(), grid, false, cs);
    }
    if (ce == cudaSuccess) {
      k_wave_cond<<<1, 1, 0, cs>>>(p->ctrl, h);
      ce = cudaGetLastError();
    }
    cudaGraph_t outg = nullptr;
    cudaError_t ee = cudaStreamEndCapture(cs, &outg);
    cudaStreamDestroy(cs);
    CUDA_TRY(p, ce);
    CUDA_TRY(p, ee);
    CUDA_TRY(p, cudaGraphInstantiate(&p->kg_exec, g, 0));
    p->kg_key = key;
  }
  CUDA_TRY(p, cudaGraphLaunch(p->kg_exec, st));
  (void)launches;  // counted from Ctrl::graph_iters after the run
  return VP_OK;
}

}  // namespace

// ====================================================================== C ABI
extern "C" {

const char* vp_status_string(vp_status s) {
  switch (s) {
    case VP_OK: return "VP_OK";
    case VP_ERR_INVALID: return "VP_ERR_INVALID";
    case VP_ERR_UNSUPPORTED: return "VP_ERR_UNSUPPORTED";
    case VP_ERR_CUDA: return "VP_ERR_CUDA";
    case VP_ERR_OOM: return "VP_ERR_OOM";
    case VP_ERR_QUEUE_OVERFLOW: return "VP_ERR_QUEUE_OVERFLOW";
    case VP_ERR_TIMEOUT: return "VP_ERR_TIMEOUT";
    case VP_ERR_BINDING: return "VP_ERR_BINDING";
    case VP_ERR_FANOUT: return "VP_ERR_FANOUT";
  }
  return "VP_ERR_UNKNOWN";
}

const char* vp_last_error(void* h) {
  vp_pipeline_s* p = (vp_pipeline_s*)h;
  return p ? p->err.c_str() : "";
}

vp_status vp_device_info(int device, int* num_sms, int* cc_major, int* cc_minor) {
  cudaDeviceProp prop;
  if (cudaGetDeviceProperties(&prop, device) != cudaSuccess) return VP_ERR_CUDA;
  if (num_sms) *num_sms = prop.multiProcessorCount;
  if (cc_major) *cc_major = prop.major;
  if (cc_minor) *cc_minor = prop.minor;
  return VP_OK;
}

vp_status vp_memcpy(void* dst, const void* src, size_t bytes, int kind, void* stream) {
  cudaMemcpyKind k = kind == 0 ? cudaMemcpyHostToDevice : kind == 1 ? cudaMemcpyDeviceToHost : cudaMemcpyDeviceToDevice;
  cudaStream_t st = (cudaStream_t)stream;
  if (cudaMemcpyAsync(dst, src, bytes, k, st) != cudaSuccess) return VP_ERR_CUDA;
  if (cudaStreamSynchronize(st) != cudaSuccess) return VP_ERR_CUDA;
  return VP_OK;
}

// Frees everything a pipeline owns; safe on a partially constructed object (every handle
// starts null), so vp_pipeline_create's error paths and vp_pipeline_destroy share it.
static void free_pipeline(vp_pipeline_s* p) {
  for (StageRec& r : p->st) {
    cudaFree(r.slots);
    cudaFree(r.seeds);
  }
  if (p->seq_arena) cudaFree(p->seq_arena);
  if (p->ctrl) cudaFree(p->ctrl);
  if (p->blk) cudaFree(p->blk);
  if (p->trace) cudaFree(p->trace);
  if (p->h_ctrl) cudaFreeHost(p->h_ctrl);
  if (p->h_blk) cudaFreeHost(p->h_blk);
  if (p->h_arrive) cudaFreeHost((void*)p->h_arrive);
  if (p->h_retire) cudaFreeHost((void*)p->h_retire);
  if (p->h_gpend) cudaFreeHost((void*)p->h_gpend);
  for (int i = 0; i < kMaxKernels; ++i) {
    if (p->streams[i]) cudaStreamDestroy(p->streams[i]);
    if (p->ev_join[i]) cudaEventDestroy(p->ev_join[i]);
    if (p->ev_kbeg[i]) cudaEventDestroy(p->ev_kbeg[i]);
  }
  if (p->kg_exec) cudaGraphExecDestroy(p->kg_exec);
  if (p->kg_graph) cudaGraphDestroy(p->kg_graph);
  for (cudaEvent_t e : p->wave_ev) cudaEventDestroy(e);
  if (p->ev_fork) cudaEventDestroy(p->ev_fork);
  if (p->ev_start) cudaEventDestroy(p->ev_start);
  if (p->ev_end) cudaEventDestroy(p->ev_end);
  delete p;
}

vp_status vp_pipeline_create(int device, const vp_pipeline_desc* d, void** out) {
  if (!out) return VP_ERR_INVALID;
  *out = nullptr;
  int ndev = 0;
  if (cudaGetDeviceCount(&ndev) != cudaSuccess || device < 0 || device >= ndev) return VP_ERR_CUDA;
  DeviceGuard dg(device);
  cudaDeviceProp prop;
  if (cudaGetDeviceProperties(&prop, device) != cudaSuccess) return VP_ERR_CUDA;
  if (prop.major < 10) return VP_ERR_UNSUPPORTED;  // sm_100a build only
  vp_pipeline_s* p = new vp_pipeline_s();
  p->device = device;
  p->num_sms = std::min(prop.multiProcessorCount, kMaxSM);
  if (d) p->desc = *d;
  if (p->desc.max_stages <= 0 || p->desc.max_stages > VP_MAX_STAGES) p->desc.max_stages = VP_MAX_STAGES;
  if (p->desc.watchdog_ms <= 0) p->desc.watchdog_ms = 30000;
  p->timeout_ms = p->desc.watchdog_ms;
  if ((p->desc.flags & VP_FLAG_TRACE) && p->desc.trace_capacity <= 0) p->desc.trace_capacity = 1 << 20;
  auto bad = [&](cudaError_t e) {
    if (e == cudaSuccess) return false;
    free_pipeline(p);
    return true;
  };
  if (bad(cudaMalloc(&p->ctrl, sizeof(Ctrl)))) return VP_ERR_OOM;
  if (bad(cudaMemset(p->ctrl, 0, sizeof(Ctrl)))) return VP_ERR_CUDA;
  if (bad(cudaMalloc(&p->blk, sizeof(uint32_t) * kMaxKernels * kMaxSM))) return VP_ERR_OOM;
  if (bad(cudaMallocHost(&p->h_ctrl, sizeof(Ctrl)))) return VP_ERR_OOM;
  if (bad(cudaMallocHost(&p->h_blk, sizeof(uint32_t) * kMaxKernels * kMaxSM))) return VP_ERR_OOM;
  {
    void* ha = nullptr;
    if (bad(cudaHostAlloc(&ha, sizeof(uint32_t) * (kMaxKernels + 1), cudaHostAllocMapped))) return VP_ERR_OOM;
    memset(ha, 0, sizeof(uint32_t) * (kMaxKernels + 1));
    p->h_arrive = (volatile uint32_t*)ha;
    if (bad(cudaHostGetDevicePointer((void**)&p->d_arrive, ha, 0))) return VP_ERR_CUDA;
    void* hr = nullptr;
    if (bad(cudaHostAlloc(&hr, sizeof(uint32_t) * kMaxKernels, cudaHostAllocMapped))) return VP_ERR_OOM;
    memset(hr, 0, sizeof(uint32_t) * kMaxKernels);
    p->h_retire = (volatile uint32_t*)hr;
    if (bad(cudaHostGetDevicePointer((void**)&p->d_retire, hr, 0))) return VP_ERR_CUDA;
    void* hg = nullptr;
    if (bad(cudaHostAlloc(&hg, sizeof(long long) * kMaxKernels * kMaxKernels, cudaHostAllocMapped))) return VP_ERR_OOM;
    memset(hg, 0, sizeof(long long) * kMaxKernels * kMaxKernels);
    p->h_gpend = (volatile long long*)hg;
    if (bad(cudaHostGetDevicePointer((void**)&p->d_gpend, hg, 0))) return VP_ERR_CUDA;
  }
  if (p->desc.flags & VP_FLAG_TRACE)
    if (bad(cudaMalloc(&p->trace, sizeof(TraceRec) * (size_t)p->desc.trace_capacity))) return VP_ERR_OOM;
  for (int i = 0; i < kMaxKernels; ++i) {
    if (bad(cudaStreamCreateWithFlags(&p->streams[i], cudaStreamNonBlocking))) return VP_ERR_CUDA;
    if (bad(cudaEventCreate(&p->ev_join[i]))) return VP_ERR_CUDA;
    if (bad(cudaEventCreate(&p->ev_kbeg[i]))) return VP_ERR_CUDA;
  }
  if (bad(cudaEventCreateWithFlags(&p->ev_fork, cudaEventDisableTiming))) return VP_ERR_CUDA;
  if (bad(cudaEventCreate(&p->ev_start)) || bad(cudaEventCreate(&p->ev_end))) return VP_ERR_CUDA;
  *out = p;
  return VP_OK;
}

vp_status vp_pipeline_destroy(void* h) {
  vp_pipeline_s* p = (vp_pipeline_s*)h;
  if (!p) return VP_ERR_INVALID;
  DeviceGuard dg(p->device);
  cudaDeviceSynchronize();
  free_pipeline(p);
  return VP_OK;
}

vp_status vp_stage_kind_info(int kind, int* item_bytes, int* threads_per_item) {
  int pos = -1;
  const FamilyOps* f = family_of_kind(kind, &pos);
  if (!f) return VP_ERR_INVALID;
  if (item_bytes) *item_bytes = f->stride(pos);
  if (threads_per_item) *threads_per_item = f->threads_per_item(pos);
  return VP_OK;
}

vp_status vp_stage_register(void* h, const vp_stage_desc* s, int* stage_id) {
  vp_pipeline_s* p = (vp_pipeline_s*)h;
  if (!p || !s) return VP_ERR_INVALID;
  if (p->queues_ready) return fail(p, VP_ERR_INVALID, "stages must be registered before vp_insert/vp_configure");
  int pos = -1;
  const FamilyOps* f = family_of_kind(s->kind, &pos);
  if (!f) return fail(p, VP_ERR_INVALID, "unknown stage kind %d", s->kind);
  if (p->fam && p->fam != f) return fail(p, VP_ERR_INVALID, "stage kind %d belongs to family '%s', pipeline is '%s'", s->kind, f->name, p->fam->name);
  if (pos != (int)p->st.size())
    return fail(p, VP_ERR_INVALID, "family '%s' stages must be registered in order: expected stage %zu, got %d", f->name, p->st.size(), pos);
  if ((int)p->st.size() >= p->desc.max_stages) return fail(p, VP_ERR_INVALID, "max_stages exceeded");
  if (s->item_bytes != f->stride(pos))
    return fail(p, VP_ERR_INVALID, "item_bytes %d != %d for stage kind %d", s->item_bytes, f->stride(pos), s->kind);
  if (s->threads_per_item != 0 && s->threads_per_item != f->threads_per_item(pos))
    return fail(p, VP_ERR_INVALID, "threads_per_item %d unsupported for kind %d (built-in uses %d)", s->threads_per_item, s->kind, f->threads_per_item(pos));
  if (s->params) {
    if (s->params_bytes != f->params_bytes()) return fail(p, VP_ERR_INVALID, "params_bytes %zu != %zu", s->params_bytes, f->params_bytes());
    std::vector<uint8_t> pr((const uint8_t*)s->params, (const uint8_t*)s->params + s->params_bytes);
    if (!p->params.empty() && p->params != pr) return fail(p, VP_ERR_INVALID, "stages of one family must share one params struct");
    p->params = pr;
  }
  p->fam = f;
  StageRec r;
  r.d = *s;
  r.name = s->name ? s->name : "";
  r.d.name = nullptr;
  int64_t cap = s->queue_capacity > 0 ? s->queue_capacity : (p->desc.default_queue_capacity > 0 ? p->desc.default_queue_capacity : (1ll << f->default_cap_log2(pos)));
  int lg = 0;
  while ((1ll << lg) < cap) ++lg;
  if (lg < 5) lg = 5;
  r.cap_log2 = lg;
  p->st.push_back(r);
  if (stage_id) *stage_id = pos;
  p->configured = false;
  return VP_OK;
}

static vp_status finish_registration(vp_pipeline_s* p) {
  if (!p->fam) return fail(p, VP_ERR_INVALID, "no stages registered");
  if ((int)p->st.size() != p->fam->S) return fail(p, VP_ERR_INVALID, "family '%s' needs all %d stages registered (%zu given)", p->fam->name, p->fam->S, p->st.size());
  if (p->params.empty()) return fail(p, VP_ERR_INVALID, "no params struct given for family '%s'", p->fam->name);
  const char* v = p->fam->validate(p->params.data());
  if (v) return fail(p, VP_ERR_INVALID, "%s", v);
  return ensure_queues(p);
}

vp_status vp_insert_async(void* h, int stage_id, const void* items, size_t n, int flags, void* stream) {
  vp_pipeline_s* p = (vp_pipeline_s*)h;
  if (!p) return VP_ERR_INVALID;
  DeviceGuard dg(p->device);
  vp_status rc = finish_registration(p);
  if (rc != VP_OK) return rc;
  if (stage_id < 0 || stage_id >= (int)p->st.size()) return fail(p, VP_ERR_INVALID, "bad stage id %d", stage_id);
  if (n > 0 && !items) return fail(p, VP_ERR_INVALID, "items is NULL");
  StageRec& r = p->st[stage_id];
  if (flags & VP_INSERT_REPLACE) r.n_seeds = 0;
  size_t stride = (size_t)p->fam->stride(stage_id);
  cudaStream_t st = (cudaStream_t)stream;
  if (r.n_seeds + n > r.seed_cap) {
    size_t ncap = std::max(r.n_seeds + n, r.seed_cap * 2);
    uint8_t* nb = nullptr;
    CUDA_TRY(p, cudaMalloc(&nb, ncap * stride));
    if (r.n_seeds) CUDA_TRY(p, cudaMemcpyAsync(nb, r.seeds, r.n_seeds * stride, cudaMemcpyDeviceToDevice, st));
    CUDA_TRY(p, cudaStreamSynchronize(st));
    cudaFree(r.seeds);
    r.seeds = nb;
    r.seed_cap = ncap;
  }
  if (n) {
    CUDA_TRY(p, cudaMemcpyAsync(r.seeds + r.n_seeds * stride, items, n * stride,
                                (flags & VP_INSERT_DEVICE) ? cudaMemcpyDeviceToDevice : cudaMemcpyHostToDevice, st));
  }
  r.n_seeds += n;
  return VP_OK;
}

vp_status vp_insert(void* h, int stage_id, const void* items, size_t n, int flags) {
  vp_pipeline_s* p = (vp_pipeline_s*)h;
  if (!p) return VP_ERR_INVALID;
  vp_status rc = vp_insert_async(h, stage_id, items, n, flags, nullptr);
  if (rc != VP_OK) return rc;
  DeviceGuard dg(p->device);
  CUDA_TRY(p, cudaStreamSynchronize(nullptr));
  return VP_OK;
}

vp_status vp_configure(void* h, int model, const vp_sm_binding* b, int batch) {
  vp_pipeline_s* p = (vp_pipeline_s*)h;
  if (!p) return VP_ERR_INVALID;
  DeviceGuard dg(p->device);
  vp_status rc = finish_registration(p);
  if (rc != VP_OK) return rc;
  if (batch < 0) return fail(p, VP_ERR_INVALID, "batch must be >= 0");
  Plan pl;
  rc = build_plan(p, model, b, batch, pl);
  if (rc != VP_OK) return rc;
  p->plan = pl;
  p->configured = true;
  return VP_OK;
}

vp_status vp_configure_config(void* h, const vp_config* c) {
  if (!c) return VP_ERR_INVALID;
  return vp_configure(h, c->model, c->has_binding ? &c->binding : nullptr, c->batch);
}

vp_status vp_get_config(void* h, vp_config* out) {
  vp_pipeline_s* p = (vp_pipeline_s*)h;
  if (!p || !out) return VP_ERR_INVALID;
  if (!p->configured) return fail(p, VP_ERR_INVALID, "not configured");
  *out = p->plan.cfg;
  return VP_OK;
}

vp_status vp_set_params(void* h, const void* params, size_t params_bytes) {
  vp_pipeline_s* p = (vp_pipeline_s*)h;
  if (!p || !params) return VP_ERR_INVALID;
  if (!p->fam) return fail(p, VP_ERR_INVALID, "vp_set_params before vp_stage_register");
  if (params_bytes != p->fam->params_bytes())
    return fail(p, VP_ERR_INVALID, "params_bytes %zu != %zu", params_bytes, p->fam->params_bytes());
  const char* v = p->fam->validate(params);
  if (v) return fail(p, VP_ERR_INVALID, "%s", v);
  p->params.assign((const uint8_t*)params, (const uint8_t*)params + params_bytes);
  return VP_OK;
}

vp_status vp_get_output(void* h, int index, void** dev_ptr, size_t* bytes) {
  vp_pipeline_s* p = (vp_pipeline_s*)h;
  if (!p || !dev_ptr || !bytes) return VP_ERR_INVALID;
  if (!p->fam || p->params.empty()) return fail(p, VP_ERR_INVALID, "no family params");
  if (!p->fam->output(p->params.data(), index, dev_ptr, bytes)) return fail(p, VP_ERR_INVALID, "no output %d", index);
  return VP_OK;
}

static vp_status run_once(vp_pipeline_s* p, cudaStream_t st, vp_run_stats* stats) {
  const int S = (int)p->st.size();
  for (int s = 0; s < S; ++s)
    if (p->run_cap_log2[s] != (p->plan.cap_log2[s] ? p->plan.cap_log2[s] : p->st[s].cap_log2)) p->dirty_queues = true;
  if (p->dirty_queues) {
    vp_status rc = reset_queues(p, st);
    if (rc != VP_OK) return rc;
  }
  RunInit ri;
  memset(&ri, 0, sizeof(ri));
  for (int s = 0; s < S; ++s) {
    ri.seeds[s] = p->st[s].n_seeds;
    ri.pending += (long long)p->st[s].n_seeds;
    if (p->plan.online && p->plan.stage_group[s] >= 0) ri.gpend[p->plan.stage_group[s]] += (long long)p->st[s].n_seeds;
  }
  ri.watchdog_ns = (unsigned long long)(p->timeout_ms * 1e6);
  p->epoch++;
  if (p->epoch == 0) p->epoch = 1;
  const Plan& pl = p->plan;
  int nk = (int)pl.kernels.size();
  // Stages no seed can reach (through the fan-out graph) never get an item: their
  // persistent kernels are not launched (they would only hold SMs, and their resident
  // idle blocks can keep a later kernel's grid from being dispatched).
  bool reach[kMaxStages] = {};
  for (int s = 0; s < S; ++s) reach[s] = p->st[s].n_seeds > 0;
  for (bool grew = true; grew;) {
    grew = false;
    for (int s = 0; s < S; ++s)
      for (int t = 0; t < S; ++t)
        if (reach[s] && !reach[t] && p->fam->fanout(s, t) > 0) reach[t] = grew = true;
  }
  uint32_t live_mask = 0;
  for (int i = 0; i < nk; ++i) {
    bool live = false;
    for (int s = pl.kernels[i].lo; s <= pl.kernels[i].hi; ++s) live |= reach[s];
    p->launched[i] = live;
    if (live) live_mask |= 1u << i;
  }
  Common c = make_common(p);
  // co-residency check only where groups depend on each other's grids being resident
  c.peer_mask = __builtin_popcount(live_mask) >= 2 ? live_mask : 0u;
  int dispatch_timeouts = 0;
  if ((p->desc.flags & VP_FLAG_L2_PERSIST) && !p->l2_window_set) {
    // keep the claim/publish sequence words in a persisting L2 carve-out
    // (the ring counters are atomics, which execute in L2 anyway)
    int max_persist = 0, max_window = 0;
    cudaDeviceGetAttribute(&max_persist, cudaDevAttrMaxPersistingL2CacheSize, p->device);
    cudaDeviceGetAttribute(&max_window, cudaDevAttrMaxAccessPolicyWindowSize, p->device);
    const size_t win = std::min(p->seq_arena_bytes, (size_t)std::max(0, max_window));
    if (max_persist > 0 && win > 0) {
      CUDA_TRY(p, cudaDeviceSetLimit(cudaLimitPersistingL2CacheSize, std::min(win, (size_t)max_persist)));
      cudaStreamAttrValue av;
      memset(&av, 0, sizeof(av));
      av.accessPolicyWindow.base_ptr = p->seq_arena;
      av.accessPolicyWindow.num_bytes = win;
      av.accessPolicyWindow.hitRatio = std::min(1.0f, (float)max_persist / (float)win);
      av.accessPolicyWindow.hitProp = cudaAccessPropertyPersisting;
      av.accessPolicyWindow.missProp = cudaAccessPropertyStreaming;
      CUDA_TRY(p, cudaStreamSetAttribute(st, cudaStreamAttributeAccessPolicyWindow, &av));
      for (int i = 0; i < kMaxKernels; ++i)
        CUDA_TRY(p, cudaStreamSetAttribute(p->streams[i], cudaStreamAttributeAccessPolicyWindow, &av));
    }
    p->l2_window_set = true;
  }
  CUDA_TRY(p, cudaEventRecord(p->ev_start, st));
  k_run_init<<<1, 256, 0, st>>>(p->ctrl, p->blk, ri);
  CUDA_TRY(p, cudaGetLastError());
  CUDA_TRY(p, p->fam->init_run(p->params.data(), st));
  const bool serialize = (p->desc.flags & VP_FLAG_SERIALIZE_GROUPS) != 0;
  if (nk > 0) {
    CUDA_TRY(p, cudaEventRecord(p->ev_fork, st));
    for (int i = 0; i < nk; ++i) {
      const KernelPlan& k = pl.kernels[i];
      cudaStream_t ks = p->streams[i];
      CUDA_TRY(p, cudaStreamWaitEvent(ks, p->ev_fork, 0));
      // test hook: each group's grid starts only after the previous one finished (what a
      // profiler's kernel serialisation does to concurrently launched groups)
      if (serialize && i > 0) CUDA_TRY(p, cudaStreamWaitEvent(ks, p->ev_join[i - 1], 0));
      const bool live = p->launched[i];
      if (!live) {
        CUDA_TRY(p, cudaEventRecord(p->ev_kbeg[i], ks));
        CUDA_TRY(p, cudaEventRecord(p->ev_join[i], ks));
        continue;
      }
      GroupArgs g;
      memset(&g, 0, sizeof(g));
      memcpy(g.sm_mask, k.mask, sizeof(g.sm_mask));
      g.quota = k.quota;
      g.kslot = k.kslot;
      g.mode = MODE_PERSISTENT;
      for (int s = 0; s < kMaxStages; ++s) g.batch[s] = pl.batch[s] ? pl.batch[s] : 1;
      g.group = pl.online ? k.group : -1;
      g.can_retire = pl.online && k.can_retire;
      g.feeders = k.feeders;
      occupancy(p, k.lo, k.hi, k.rtc);
      CUDA_TRY(p, cudaEventRecord(p->ev_kbeg[i], ks));
      CUDA_TRY(p, p->fam->launch(k.lo, k.hi, k.rtc, c, g, p->params.data(), k.grid, k.coop, ks));
      CUDA_TRY(p, cudaEventRecord(p->ev_join[i], ks));
      if (i + 1 < nk) {
        // High-level control: launch the next group's kernel only after this grid is
        // fully dispatched, so its admitted blocks hold their SMs before the next
        // kernel's blocks arrive (deterministic filling-retreating, L27 §5).
        auto t0 = std::chrono::steady_clock::now();
        while (p->h_arrive[i] != p->epoch) {
          if (p->h_arrive[kMaxKernels] == p->epoch) break;  // aborted: groups not co-resident
          if (std::chrono::steady_clock::now() - t0 > std::chrono::milliseconds(2000)) {
            // binding is then no longer deterministic (the next grid may take SMs this one
            // wanted); recorded in vp_run_stats.dispatch_timeouts
            ++dispatch_timeouts;
            break;
          }
        }
      }
    }
  }
  int nk_total = nk;
  if (pl.online) {
    // Online adaptation: when a group retires (its last block left: mapped flag), launch
    // a refill grid of its downstream group restricted to the freed SMs.
    bool handled[kMaxKernels] = {};
    for (;;) {
      bool running = false;
      for (int i = 0; i < nk_total; ++i) {
        cudaError_t q = cudaEventQuery(p->ev_join[i]);
        if (q == cudaErrorNotReady) running = true;
        else if (q != cudaSuccess) CUDA_TRY(p, q);
      }
      if (!running) break;
      for (int i = 0; i < nk; ++i) {
        const KernelPlan& k = pl.kernels[i];
        if (handled[i] || k.refill < 0 || p->h_retire[i] != p->epoch || nk_total >= kMaxKernels) continue;
        handled[i] = true;
        // the freed SMs go to the group that has the most stalled items at
        // that moment (the retiring block's snapshot of every group's alive count); the
        // first downstream group when none has any
        int pick = k.refill;
        long long most = 0;
        for (uint32_t m = k.refill_cands; m; m &= m - 1) {
          const int j = __builtin_ctz(m);
          const long long alive = p->h_gpend[i * kMaxKernels + pl.kernels[j].group];
          if (alive > most) {
            most = alive;
            pick = j;
          }
        }
        p->refill_pick[i] = pick;
        const KernelPlan& t = pl.kernels[pick];
        const int slot = nk_total++;
        GroupArgs g;
        memset(&g, 0, sizeof(g));
        memcpy(g.sm_mask, k.mask, sizeof(g.sm_mask));  // the retired group's SMs
        g.quota = t.quota;
        g.kslot = slot;
        g.mode = MODE_PERSISTENT;
        for (int s = 0; s < kMaxStages; ++s) g.batch[s] = pl.batch[s] ? pl.batch[s] : 1;
        g.group = t.group;
        g.can_retire = t.can_retire;
        g.feeders = t.feeders;
        const int per = t.quota > 0 ? t.quota : std::max(1, occupancy(p, t.lo, t.hi, t.rtc));
        const int grid = per * std::max(1, mask_count(k.mask, p->num_sms));
        cudaStream_t ks = p->streams[slot];
        CUDA_TRY(p, cudaEventRecord(p->ev_kbeg[slot], ks));
        CUDA_TRY(p, p->fam->launch(t.lo, t.hi, t.rtc, c, g, p->params.data(), grid, false, ks));
        CUDA_TRY(p, cudaEventRecord(p->ev_join[slot], ks));
        p->refill_lo[slot] = t.lo;
        p->refill_hi[slot] = t.hi;
        p->refill_quota[slot] = t.quota;
      }
      std::this_thread::yield();
    }
  }
  uint64_t launches = 0;
  p->wave_stage.clear();
  if (pl.kbk_graph) {
    vp_status rc = graph_wave_run(p, c, st, &launches);
    if (rc != VP_OK) return rc;
  } else if (!pl.kbk_stages.empty() || pl.wave_rtc) {
    vp_status rc = host_wave_loop(p, c, st, &launches);
    if (rc != VP_OK) return rc;
  }
  for (int i = 0; i < nk_total; ++i) CUDA_TRY(p, cudaStreamWaitEvent(st, p->ev_join[i], 0));
  CUDA_TRY(p, p->fam->finalize(p->params.data(), st));
  CUDA_TRY(p, cudaEventRecord(p->ev_end, st));
  CUDA_TRY(p, cudaMemcpyAsync(p->h_ctrl, p->ctrl, sizeof(Ctrl), cudaMemcpyDeviceToHost, st));
  CUDA_TRY(p, cudaMemcpyAsync(p->h_blk, p->blk, sizeof(uint32_t) * kMaxKernels * kMaxSM, cudaMemcpyDeviceToHost, st));
  CUDA_TRY(p, cudaStreamSynchronize(st));
  float ms = 0;
  cudaEventElapsedTime(&ms, p->ev_start, p->ev_end);
  const Ctrl& hc = *p->h_ctrl;
  if (stats) {
    memset(stats, 0, sizeof(*stats));
    stats->device_ms = ms;
    for (int s = 0; s < S; ++s) {
      stats->dequeued[s] = hc.deq[s];
      stats->enqueued[s] = hc.enq[s];
      stats->max_depth[s] = hc.max_depth[s];
    }
    stats->num_kernels = nk_total;  // + refill grids of the online adaptation
    for (int i = 0; i < nk_total && i < 16; ++i) {
      stats->kernel_lo[i] = i < nk ? pl.kernels[i].lo : p->refill_lo[i];
      stats->kernel_hi[i] = i < nk ? pl.kernels[i].hi : p->refill_hi[i];
      stats->kernel_quota[i] = i < nk ? pl.kernels[i].quota : p->refill_quota[i];
      float kms = 0;
      cudaEventElapsedTime(&kms, p->ev_kbeg[i], p->ev_join[i]);
      stats->kernel_ms[i] = kms;
      stats->admitted[i] = hc.admitted[i].v;
      for (int sm = 0; sm < VP_MAX_SM; ++sm) stats->blocks_on_sm[i][sm] = p->h_blk[i * kMaxSM + sm];
    }
    if (nk == 0) {
      for (int sm = 0; sm < VP_MAX_SM; ++sm) stats->blocks_on_sm[0][sm] = p->h_blk[sm];
    }
    stats->fallback_admits = hc.fallback_admits;
    stats->kbk_launches = pl.kbk_graph ? hc.graph_iters * pl.kbk_stages.size() : launches;
    stats->trace_records = hc.trace_n.v;
    stats->abort_reason = (int)hc.abort.v;
    stats->num_sms = p->num_sms;
    for (int s = 0; s < S; ++s) {
      stats->stage_exec_ns[s] = hc.exec_ns[s];
      stats->stage_flush_ns[s] = hc.flush_ns[s];
    }
    for (int i = 0; i < kMaxKernels; ++i) {
      stats->kernel_idle_ns[i] = hc.idle_ns[i];
      stats->kernel_rounds[i] = hc.rounds[i];
    }
    for (size_t w = 0; w < p->wave_stage.size(); ++w) {
      float ms_w = 0.0f;
      if (cudaEventElapsedTime(&ms_w, p->wave_ev[2 * w], p->wave_ev[2 * w + 1]) == cudaSuccess)
        stats->stage_wave_ms[p->wave_stage[w]] += ms_w;
    }
    for (int s = 0; s < S; ++s) {
      stats->ring_tail[s] = hc.tail[s].v;
      stats->ring_head[s] = hc.head[s].v;
      stats->ring_count[s] = (int64_t)hc.count[s].v;
      stats->seed_head[s] = hc.seed_head[s].v;
    }
    stats->pending = (int64_t)hc.pending.v;
    stats->dispatch_timeouts = dispatch_timeouts;
    for (int s = 0; s < S; ++s) stats->work_units[s] = hc.units[s];
    for (int s = 0; s < S; ++s) stats->stolen[s] = hc.stolen[s];
    stats->model_rerun = 0;
  }
  if (hc.abort.v != ABORT_NONE) {
    p->dirty_queues = true;
    switch (hc.abort.v) {
      case ABORT_TIMEOUT: return fail(p, VP_ERR_TIMEOUT, "device watchdog fired after %.3f ms", p->timeout_ms);
      case ABORT_OVERFLOW: return fail(p, VP_ERR_QUEUE_OVERFLOW, "a ring stayed full for > 200 ms (raise queue_capacity)");
      case ABORT_FANOUT: return fail(p, VP_ERR_FANOUT, "a stage exceeded its declared fan-out");
      case ABORT_GUARD: return fail(p, VP_ERR_INVALID, "a stage's recursion guard fired (input outside the domain)");
      case ABORT_NOT_CORESIDENT:
        return fail(p, VP_ERR_UNSUPPORTED, "a planned group's grid never became resident while another group waited on it "
                                           "(non-concurrent kernel scheduling: profiler, MPS or a co-tenant)");
      default: return fail(p, VP_ERR_CUDA, "unknown abort reason %llu", (unsigned long long)hc.abort.v);
    }
  }
  if ((long long)hc.pending.v != 0) {
    p->dirty_queues = true;
    return fail(p, VP_ERR_CUDA, "pipeline ended with pending = %lld", (long long)hc.pending.v);
  }
  if (p->desc.flags & VP_FLAG_STRICT_BINDING) {
    for (int i = 0; i < nk; ++i) {
      const KernelPlan& k = pl.kernels[i];
      if (k.quota <= 0 || !p->launched[i]) continue;
      for (int sm = 0; sm < p->num_sms; ++sm)
        if ((k.mask[sm >> 5] >> (sm & 31)) & 1u)
          if ((int)p->h_blk[i * kMaxSM + sm] < k.quota)
            return fail(p, VP_ERR_BINDING, "kernel %d reached %u of %d blocks on SM %d", i, p->h_blk[i * kMaxSM + sm], k.quota, sm);
    }
  }
  return VP_OK;
}

vp_status vp_run(void* h, void* stream, vp_run_stats* stats) {
  vp_pipeline_s* p = (vp_pipeline_s*)h;
  if (!p) return VP_ERR_INVALID;
  if (!p->configured) return fail(p, VP_ERR_INVALID, "vp_run before vp_configure/vp_autotune");
  DeviceGuard dg(p->device);
  cudaStream_t st = (cudaStream_t)stream;
  vp_status rc = run_once(p, st, stats);
  if (rc != VP_ERR_UNSUPPORTED || p->h_ctrl->abort.v != ABORT_NOT_CORESIDENT || (p->desc.flags & VP_FLAG_NO_RERUN))
    return rc;
  // The groups of this plan could not all be resident at once: the run is
  // repeated from its seeds as one cooperative megakernel, which the driver co-schedules by
  // construction; every model computes the same result (SURVEY §8(c-6) model equivalence).
  const double first_ms = stats ? stats->device_ms : 0.0;
  Plan saved = p->plan;
  Plan mega;
  rc = build_plan(p, VP_MEGAKERNEL, nullptr, saved.cfg.batch, mega);
  if (rc != VP_OK) return rc;
  p->plan = mega;
  p->dirty_queues = true;  // the aborted run's rings are reset before the rerun
  rc = run_once(p, st, stats);
  p->plan = saved;
  p->dirty_queues = true;
  if (stats) {
    stats->device_ms += first_ms;
    stats->model_rerun = 1;
  }
  return rc;
}

vp_status vp_get_trace(void* h, void** dev_ptr, size_t* n) {
  vp_pipeline_s* p = (vp_pipeline_s*)h;
  if (!p || !dev_ptr || !n) return VP_ERR_INVALID;
  if (!(p->desc.flags & VP_FLAG_TRACE)) return fail(p, VP_ERR_INVALID, "pipeline created without VP_FLAG_TRACE");
  *dev_ptr = p->trace;
  unsigned long long m = p->h_ctrl ? p->h_ctrl->trace_n.v : 0;
  *n = (size_t)std::min<unsigned long long>(m, (unsigned long long)p->desc.trace_capacity);
  return VP_OK;
}

// ---- internal accessors for the auto-tuner (vp_tune.cu); not part of vp.h
int vpi_num_stages(void* h) { return h ? (int)((vp_pipeline_s*)h)->st.size() : 0; }
int vpi_num_sms(void* h) { return h ? ((vp_pipeline_s*)h)->num_sms : 0; }
int vpi_rtc_legal(void* h, int lo, int hi) {
  vp_pipeline_s* p = (vp_pipeline_s*)h;
  return p && p->fam && p->fam->rtc_legal(lo, hi) ? 1 : 0;
}
int vpi_default_batch(void* h, int s) { return ((vp_pipeline_s*)h)->fam->default_batch(s); }
vp_status vp_set_flags(void* h, uint32_t flags, uint32_t* old_flags) {
  vp_pipeline_s* p = (vp_pipeline_s*)h;
  if (!p) return VP_ERR_INVALID;
  const uint32_t mutable_bits =
      VP_FLAG_QUEUE_DEPTH | VP_FLAG_STRICT_BINDING | VP_FLAG_TIMERS | VP_FLAG_SERIALIZE_GROUPS | VP_FLAG_NO_RERUN |
      VP_FLAG_CLUSTER_STEAL;
  if (flags & ~mutable_bits)
    return fail(p, VP_ERR_INVALID,
                "vp_set_flags: only QUEUE_DEPTH, STRICT_BINDING, TIMERS, SERIALIZE_GROUPS, NO_RERUN, CLUSTER_STEAL change after create");
  if (old_flags) *old_flags = p->desc.flags;
  p->desc.flags = (p->desc.flags & ~mutable_bits) | flags;
  return VP_OK;
}

uint32_t vpi_swap_flags(void* h, uint32_t flags) {
  vp_pipeline_s* p = (vp_pipeline_s*)h;
  uint32_t old = p->desc.flags;
  p->desc.flags = flags;
  return old;
}
double vpi_timeout(void* h) { return ((vp_pipeline_s*)h)->timeout_ms; }
void vpi_set_error(void* h, const char* msg) { ((vp_pipeline_s*)h)->err = msg; }

vp_status vp_set_timeout(void* h, double ms) {
  vp_pipeline_s* p = (vp_pipeline_s*)h;
  if (!p || !(ms > 0)) return VP_ERR_INVALID;
  p->timeout_ms = ms;
  return VP_OK;
}

vp_status vp_profile(void* h, int* max_blocks, int* regs, int* smem) {
  vp_pipeline_s* p = (vp_pipeline_s*)h;
  if (!p) return VP_ERR_INVALID;
  DeviceGuard dg(p->device);
  vp_status rc = finish_registration(p);
  if (rc != VP_OK) return rc;
  for (int s = 0; s < (int)p->st.size(); ++s) {
    const void* fn = p->fam->kernel(s, s, false);
    cudaFuncAttributes at;
    CUDA_TRY(p, cudaFuncGetAttributes(&at, fn));
    if (max_blocks) max_blocks[s] = occupancy(p, s, s, false);
    if (regs) regs[s] = at.numRegs;
    if (smem) smem[s] = (int)(at.sharedSizeBytes + p->fam->smem(s, s, false));
  }
  return VP_OK;
}

}  // extern "C"

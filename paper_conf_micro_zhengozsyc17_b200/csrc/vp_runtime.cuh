// vp_runtime.cuh — device side of the VersaPipe runtime for sm_100a.
//
// One template kernel realises every execution model of PAPER.md §4 (L11–L27):
//   * persistent threads (L13, L17): blocks loop "fetch item batch -> execute -> push"
//     until the pipeline drains (pending == 0);
//   * Megakernel (L13 Fig. 3c): one kernel over all stages, blocks "query queues in turn
//     of priority" (Fig. 8a, L31/L37);
//   * coarse / fine pipeline (L21 Figs. 4–5): one persistent kernel per stage, bound to
//     SMs by check_sm() and to per-(stage,SM) block quotas by check_sm_blk();
//   * RTC (L11): all stages of a linear group in one kernel, intermediate items passed
//     block-locally in shared memory instead of through work queues;
//   * KBK (L13 Fig. 3b): the same kernel in non-persistent "wave" mode, one launch per
//     stage over the items present, driven by the host.
//
// B200-first mechanics: per-stage bounded MPMC rings with 64-bit
// tickets and per-slot sequence words (Vyukov), block-aggregated claims and publishes
// (2 L2 atomics per block batch per queue), one pending-counter atomic per batch,
// 16-B (or 4/8-B for small items) coalesced payload movement through shared memory,
// L1-bypassing (.cg) payload loads, release/acquire publication, %smid binding,
// %globaltimer watchdog.
#pragma once
#include <cuda_runtime.h>
#include <stdint.h>

#include <type_traits>
#include <utility>

namespace vp {

constexpr int kThreads = 256;       // worker threads per block: the paper's block size (L53)
constexpr int kWarpsW = kThreads / 32;
constexpr int kBlock = kThreads + 64;  // + a fetcher warp and a publisher warp (task scheduler)
constexpr int kMaxStages = 8;
constexpr int kMaxKernels = 16;     // kernel slots per run (binding counters)
constexpr int kMaxSM = 256;         // table width; B200 has 148 SMs (queried at runtime)
constexpr int kMaskWords = kMaxSM / 32;

enum Abort : unsigned long long {
  ABORT_NONE = 0,
  ABORT_TIMEOUT = 1,   // watchdog deadline passed (VP_ERR_TIMEOUT)
  ABORT_OVERFLOW = 2,  // a producer could not get a free ring slot (VP_ERR_QUEUE_OVERFLOW)
  ABORT_FANOUT = 3,    // a stage emitted more items than its declared fan-out
  ABORT_GUARD = 4,     // a stage's own recursion guard fired (invalid input)
  ABORT_NOT_CORESIDENT = 5,  // a group waited on a planned group whose grid never became
                             // resident (non-concurrent scheduling: profiler, MPS, co-tenant)
};

// Each hot counter on its own 128-B line (no false sharing between L2 atomics).
struct alignas(128) Line {
  unsigned long long v;
  unsigned long long pad[15];
};

struct Ctrl {
  Line tail[kMaxStages];       // producer reservation ticket
  Line head[kMaxStages];       // consumer claim ticket
  Line count[kMaxStages];      // published-and-unclaimed items (signed)
  Line seed_head[kMaxStages];  // claim index into the seed segment
  Line pending;                // items alive: seeded + emitted - completed (signed)
  Line abort;                  // Abort reason, first writer wins
  Line deadline;               // %globaltimer deadline in ns
  Line trace_n;
  Line arrivals[kMaxKernels];  // blocks of each kernel that ran the binding prologue
  Line admitted[kMaxKernels];  // blocks of each kernel that stayed
  unsigned long long deq[kMaxStages];
  unsigned long long enq[kMaxStages];      // includes seeds
  unsigned long long max_depth[kMaxStages];
  unsigned long long fallback_admits;
  unsigned long long exec_ns[kMaxStages];   // FLAG_TIMERS: stage-in + execute per stage
  unsigned long long flush_ns[kMaxStages];  // FLAG_TIMERS: publish (queue overhead) per stage
  unsigned long long idle_ns[kMaxKernels];  // FLAG_TIMERS: blocks finding no work, per kernel
  unsigned long long rounds[kMaxKernels];   // persistent-loop rounds, summed over blocks, per kernel
  unsigned long long units[kMaxStages];     // family-defined work units per stage (vp_run_stats.work_units)
  Line gpend[kMaxKernels];                  // online adaptation: items alive in each group's stages
  unsigned long long retired[kMaxKernels];  // online adaptation: group drained for good, its blocks exit
  unsigned long long exits[kMaxKernels];    // admitted blocks of each kernel slot that have exited
  unsigned long long graph_iters;           // device-driven KBK: iterations of the graph's while loop
  long long wave_n[kMaxStages];             // device-driven KBK: size of each stage's current wave
  unsigned long long stolen[kMaxStages];    // cluster work stealing: items taken from a sibling's queue
};

struct QueueDesc {
  uint8_t* slots;            // [cap][stride]
  unsigned long long* seq;   // [cap]
  const uint8_t* seeds;      // [n_seeds][stride] (read-only during a run)
  long long n_seeds;
  uint32_t cap_log2;
  uint32_t stride;
};

struct TraceRec {
  unsigned long long id;
  uint32_t stage, smid;
  uint32_t kslot, block;  // kernel slot and blockIdx.x of the executing block (binding checks)
};

enum : uint32_t { FLAG_TRACE = 1u, FLAG_DEPTH = 2u, FLAG_TIMERS = 4u, FLAG_STEAL = 8u };

// ------------------------------------------------------------------ thread-block clusters
// (cluster-local queues over distributed shared memory)
__device__ __forceinline__ uint32_t cluster_ctarank() {
  uint32_t r;
  asm volatile("mov.u32 %0, %%cluster_ctarank;" : "=r"(r));
  return r;
}
__device__ __forceinline__ uint32_t cluster_nctarank() {
  uint32_t r;
  asm volatile("mov.u32 %0, %%cluster_nctarank;" : "=r"(r));
  return r;
}
// shared::cluster address of `p` (this CTA's shared memory) in the CTA of cluster rank `rank`
__device__ __forceinline__ uint32_t dsmem_addr(const void* p, uint32_t rank) {
  const uint32_t a = (uint32_t)__cvta_generic_to_shared(p);
  uint32_t r;
  asm volatile("mapa.shared::cluster.u32 %0, %1, %2;" : "=r"(r) : "r"(a), "r"(rank));
  return r;
}
__device__ __forceinline__ void cluster_sync_all() {
  asm volatile("barrier.cluster.arrive.release.aligned;\n\tbarrier.cluster.wait.acquire.aligned;" ::: "memory");
}
__device__ __forceinline__ bool dsmem_trylock(uint32_t addr) {
  uint32_t old;
  asm volatile("atom.acquire.cluster.shared::cluster.cas.b32 %0, [%1], 0, 1;" : "=r"(old) : "r"(addr) : "memory");
  return old == 0;
}
__device__ __forceinline__ void dsmem_st_release(uint32_t addr, int v) {
  asm volatile("st.release.cluster.shared::cluster.b32 [%0], %1;" ::"r"(addr), "r"(v) : "memory");
}
__device__ __forceinline__ int dsmem_ld_acquire(uint32_t addr) {
  int v;
  asm volatile("ld.acquire.cluster.shared::cluster.b32 %0, [%1];" : "=r"(v) : "r"(addr) : "memory");
  return v;
}
__device__ __forceinline__ int dsmem_ld_relaxed(uint32_t addr) {
  int v;
  asm volatile("ld.relaxed.cluster.shared::cluster.b32 %0, [%1];" : "=r"(v) : "r"(addr) : "memory");
  return v;
}
__device__ __forceinline__ uint4 dsmem_ld_v4(uint32_t addr) {
  uint4 v;
  asm volatile("ld.shared::cluster.v4.u32 {%0, %1, %2, %3}, [%4];" : "=r"(v.x), "=r"(v.y), "=r"(v.z), "=r"(v.w) : "r"(addr) : "memory");
  return v;
}
__device__ __forceinline__ uint32_t dsmem_ld_u32(uint32_t addr) {
  uint32_t v;
  asm volatile("ld.shared::cluster.u32 %0, [%1];" : "=r"(v) : "r"(addr) : "memory");
  return v;
}
__device__ __forceinline__ void fence_acq_rel_cluster() { asm volatile("fence.acq_rel.cluster;" ::: "memory"); }
template <class V>
__device__ __forceinline__ V dsmem_ld(uint32_t addr) {
  if constexpr (sizeof(V) == 16) {
    const uint4 v = dsmem_ld_v4(addr);
    return *(const V*)&v;
  } else if constexpr (sizeof(V) == 8) {
    uint2 v;
    asm volatile("ld.shared::cluster.v2.u32 {%0, %1}, [%2];" : "=r"(v.x), "=r"(v.y) : "r"(addr) : "memory");
    return *(const V*)&v;
  } else {
    const uint32_t v = dsmem_ld_u32(addr);
    return *(const V*)&v;
  }
}

struct Common {
  QueueDesc q[kMaxStages];
  Ctrl* ctrl;
  uint32_t* blk;             // [kMaxKernels][kMaxSM] per-(kernel, SM) block counters (D4)
  TraceRec* trace;
  unsigned long long trace_cap;
  uint32_t flags;
  int n_stages;
  volatile uint32_t* host_arrive;  // mapped pinned host words: grid of kernel k fully dispatched;
                                   // [kMaxKernels]: the run aborted as not co-resident
  volatile uint32_t* host_retire;  // mapped pinned host words: every block of kernel k exited on retirement
  volatile long long* host_gpend;  // mapped pinned [kMaxKernels][kMaxKernels]: every group's alive count,
                                   // snapshotted when kernel k retires (the host's refill choice)
  uint32_t epoch;                  // run counter written into host_arrive / host_retire
  int8_t stage_group[kMaxStages];  // online adaptation: group of each stage (-1: none / KBK)
  uint32_t peer_mask;              // planned persistent kernel slots of this run: a block stalled
                                   // for > kCoresidentNs while one of them has no block resident
                                   // aborts with ABORT_NOT_CORESIDENT
};
constexpr unsigned long long kCoresidentNs = 20000000ull;  // 20 ms

enum : int { MODE_PERSISTENT = 0, MODE_WAVE = 1 };

struct GroupArgs {
  uint32_t sm_mask[kMaskWords];  // s_flag(group, sm) (Fig. 5, L21)
  int quota;                     // blocks per SM (check_sm_blk threshold), <= 0: no cap
  int kslot;                     // kernel slot for the binding counters
  int mode;                      // MODE_PERSISTENT or MODE_WAVE
  int wave_stage;                // WAVE: the stage whose items this launch processes
  long long wave_n;              // WAVE: number of items in this launch
  long long wave_chunk;          // WAVE: items per block (a multiple of the batch)
  const long long* wave_n_dev;   // WAVE, device-driven KBK: wave size written by the planner
                                 // kernel just before this launch (overrides wave_n/chunk)
  int batch[kMaxStages];         // items per claim, per stage
  // online adaptation (the online tuner adjusts SM mappings at run time):
  // a group whose stages can receive no more items (its feeders retired, gpend == 0)
  // retires, and the host gives its SMs to another group
  int group;                     // group id of this kernel (-1: no adaptation)
  int can_retire;
  uint32_t feeders;              // bitmask of the groups that emit into this group's stages
};

template <class F>
struct KArgs {
  Common c;
  GroupArgs g;
  typename F::Params p;
};

// ------------------------------------------------------------------ PTX helpers
__device__ __forceinline__ uint32_t smid() {
  uint32_t r;
  asm volatile("mov.u32 %0, %%smid;" : "=r"(r));
  return r;
}
__device__ __forceinline__ unsigned long long globaltimer() {
  unsigned long long t;
  asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
  return t;
}
__device__ __forceinline__ unsigned long long ld_acquire(const unsigned long long* p) {
  unsigned long long v;
  asm volatile("ld.acquire.gpu.global.u64 %0, [%1];" : "=l"(v) : "l"(p) : "memory");
  return v;
}
__device__ __forceinline__ unsigned long long ld_relaxed(const unsigned long long* p) {
  unsigned long long v;
  asm volatile("ld.relaxed.gpu.global.u64 %0, [%1];" : "=l"(v) : "l"(p) : "memory");
  return v;
}
__device__ __forceinline__ void st_release(unsigned long long* p, unsigned long long v) {
  asm volatile("st.release.gpu.global.u64 [%0], %1;" ::"l"(p), "l"(v) : "memory");
}
__device__ __forceinline__ void st_relaxed(unsigned long long* p, unsigned long long v) {
  asm volatile("st.relaxed.gpu.global.u64 [%0], %1;" ::"l"(p), "l"(v) : "memory");
}
__device__ __forceinline__ unsigned long long atom_add(unsigned long long* p, long long d) {
  return atomicAdd(p, (unsigned long long)d);
}
__device__ __forceinline__ void red_add(unsigned long long* p, long long d) {
  asm volatile("red.relaxed.gpu.global.add.u64 [%0], %1;" ::"l"(p), "l"((unsigned long long)d) : "memory");
}
__device__ __forceinline__ void fence_acq_rel_gpu() { asm volatile("fence.acq_rel.gpu;" ::: "memory"); }

// Bulk (TMA, non-tensor) copies between global memory and shared memory (sm_90+).
// Ring ranges are contiguous up to the wrap point, so one claimed batch moves with one
// or two instructions issued by one thread instead of ~n*stride/16 per-lane accesses.
__device__ __forceinline__ uint32_t smem_u32(const void* p) { return (uint32_t)__cvta_generic_to_shared(p); }
__device__ __forceinline__ void mbar_init(unsigned long long* m, uint32_t count) {
  asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(smem_u32(m)), "r"(count) : "memory");
  asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
}
__device__ __forceinline__ void mbar_arrive_expect_tx(unsigned long long* m, uint32_t bytes) {
  asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(smem_u32(m)), "r"(bytes) : "memory");
}
__device__ __forceinline__ void mbar_arrive(unsigned long long* m) {
  asm volatile("mbarrier.arrive.release.cta.shared::cta.b64 _, [%0];" ::"r"(smem_u32(m)) : "memory");
}
__device__ __forceinline__ void mbar_wait(unsigned long long* m, uint32_t parity) {
  uint32_t done = 0;
  while (!done) {
    asm volatile(
        "{\n\t.reg .pred p;\n\t"
        "mbarrier.try_wait.parity.shared::cta.b64 p, [%1], %2;\n\t"
        "selp.u32 %0, 1, 0, p;\n\t}"
        : "=r"(done)
        : "r"(smem_u32(m)), "r"(parity)
        : "memory");
  }
}
// Worker-side wait on a buffer hand-over: the warp is suspended in the barrier (up to the
// time hint) instead of re-issuing try_wait, so idle workers leave the issue slots to the
// warps that still execute.
// The suspend hint alone returns often (round 2 profile: the retry loop was 5.4% of the
// fused [Dice, Shade] kernel's executed instructions).  kMaxNs > 0 adds an exponential
// __nanosleep back-off after a failed try_wait (capped at kMaxNs).  Measured on config 5:
// no gain for the fused [Dice, Shade] kernel (256 / 1024 ns: within +-0.5%), so only the
// direct-publish kernels ([Bound, Split]) use it, VP_BS_BACKOFF_NS.
#ifndef VP_MBAR_NS
#define VP_MBAR_NS 0
#endif
#ifndef VP_BS_BACKOFF_NS
#define VP_BS_BACKOFF_NS 0
#endif
template <int kMaxNs = VP_MBAR_NS>
__device__ __forceinline__ void mbar_wait_sleep(unsigned long long* m, uint32_t parity) {
  uint32_t done = 0;
  uint32_t ns = 32;
  for (;;) {
    asm volatile(
        "{\n\t.reg .pred p;\n\t"
        "mbarrier.try_wait.parity.shared::cta.b64 p, [%1], %2, %3;\n\t"
        "selp.u32 %0, 1, 0, p;\n\t}"
        : "=r"(done)
        : "r"(smem_u32(m)), "r"(parity), "r"(20000u)
        : "memory");
    if (done) break;
    if (kMaxNs > 0) {
      __nanosleep(ns);
      ns = ns * 2 < (uint32_t)kMaxNs ? ns * 2 : (uint32_t)kMaxNs;
    }
  }
}
__device__ __forceinline__ void bulk_g2s(void* dst, const void* src, uint32_t bytes, unsigned long long* m) {
  asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(
                   smem_u32(dst)),
               "l"(src), "r"(bytes), "r"(smem_u32(m))
               : "memory");
}
__device__ __forceinline__ void bulk_s2g(void* dst, const void* src, uint32_t bytes) {
  asm volatile("cp.async.bulk.global.shared::cta.bulk_group [%0], [%1], %2;" ::"l"(dst), "r"(smem_u32(src)), "r"(bytes)
               : "memory");
}
__device__ __forceinline__ void bulk_commit_wait_all() {
  asm volatile("cp.async.bulk.commit_group;" ::: "memory");
  asm volatile("cp.async.bulk.wait_group 0;" ::: "memory");
}
// generic-proxy shared-memory writes -> later async-proxy (bulk) reads of them
__device__ __forceinline__ void fence_proxy_async_smem() { asm volatile("fence.proxy.async.shared::cta;" ::: "memory"); }
// async-proxy global writes/reads <-> generic-proxy release/acquire on the slot sequence words
__device__ __forceinline__ void fence_proxy_async_global() { asm volatile("fence.proxy.async.global;" ::: "memory"); }

// Vector chunk used to move items of a given stride (16 B when possible).
template <int STRIDE>
struct Chunk {
  static constexpr int bytes = (STRIDE % 16 == 0) ? 16 : (STRIDE % 8 == 0) ? 8 : 4;
  using T = typename std::conditional<bytes == 16, uint4, typename std::conditional<bytes == 8, uint2, uint32_t>::type>::type;
  static constexpr int per_item = STRIDE / bytes;
};
template <class T>
__device__ __forceinline__ T ld_cg(const T* p) { return __ldcg(p); }
template <class T>
__device__ __forceinline__ void st_cg(T* p, T v) { __stcg(p, v); }

// A family may run an RTC chain [s, hi] itself (F::fused_rtc(s, hi) and
// F::exec_rtc_chain<s, hi>), e.g. with warp-granular hand-off instead of block barriers.
template <class F, class = void>
struct HasFusedRtc : std::false_type {};
template <class F>
struct HasFusedRtc<F, std::void_t<decltype(F::fused_rtc(0, 0))>> : std::true_type {};
template <class F, bool kHas = HasFusedRtc<F>::value>
struct FusedChain {
  template <int S0, int HI, class C>
  static __device__ __forceinline__ void run(C&, const uint8_t*, int) {}
};
template <class F>
struct FusedChain<F, true> {
  template <int S0, int HI, class C>
  static __device__ __forceinline__ void run(C& ctx, const uint8_t* items, int n) {
    F::template exec_rtc_chain<S0, HI>(ctx, items, n);
  }
};
template <class F>
constexpr bool fused_chain(int s, int hi) {
  if constexpr (HasFusedRtc<F>::value) return F::fused_rtc(s, hi);
  else return false;
}

// A family may cap a stage's batch per kernel (F::kernel_max_batch(lo, hi, rtc, s)),
// e.g. a larger batch only where its outputs stay block-local; default F::max_batch(s).
template <class F, class = void>
struct HasKernelMaxBatch : std::false_type {};
template <class F>
struct HasKernelMaxBatch<F, std::void_t<decltype(F::kernel_max_batch(0, 0, false, 0))>> : std::true_type {};
template <class F>
constexpr int kernel_max_batch(int lo, int hi, bool rtc, int s) {
  if constexpr (HasKernelMaxBatch<F>::value) return F::kernel_max_batch(lo, hi, rtc, s);
  else return F::max_batch(s);
}
// A family may size its shared-memory scratch per kernel kind (F::scratch_bytes_k(lo, hi,
// rtc)), e.g. scratch only an RTC chain uses; default F::scratch_bytes(lo, hi).
template <class F, class = void>
struct HasScratchK : std::false_type {};
template <class F>
struct HasScratchK<F, std::void_t<decltype(F::scratch_bytes_k(0, 0, false))>> : std::true_type {};
template <class F>
constexpr int scratch_of(int lo, int hi, bool rtc) {
  if constexpr (HasScratchK<F>::value) return F::scratch_bytes_k(lo, hi, rtc);
  else return F::scratch_bytes(lo, hi);
}

// A family may let the two CTAs of a thread-block cluster take items from each other's
// block-local queues over distributed shared memory (F::kClusterSteal).
// Active only when the kernel was launched as clusters of 2 (the host does that for a
// cooperative megakernel with VP_FLAG_CLUSTER_STEAL).
template <class F, class = void>
struct HasClusterSteal : std::false_type {};
template <class F>
struct HasClusterSteal<F, std::void_t<decltype(F::kClusterSteal)>> : std::bool_constant<F::kClusterSteal> {};

template <class F>
constexpr int fused_local_cap(int lo, int hi, int t) {
  if constexpr (HasFusedRtc<F>::value) return F::fused_local_cap(lo, hi, t);
  else return 0;
}

// A family may run the batches of a persistent (non-RTC) kernel [lo, hi] with block-local
// recursion (F::local_recursion(lo, hi), F::exec_local<s, LO, HI>): children that would go
// back to a ring of the same kernel are processed in the block from a shared-memory work
// stack, and only what does not fit is published.  Its out-buffer capacities are then
// F::local_out_cap(lo, hi, t).
template <class F, class = void>
struct HasLocalRec : std::false_type {};
template <class F>
struct HasLocalRec<F, std::void_t<decltype(F::local_recursion(0, 0))>> : std::true_type {};
template <class F>
constexpr bool local_recursion(int lo, int hi, bool rtc) {
  if constexpr (HasLocalRec<F>::value) return !rtc && F::local_recursion(lo, hi);
  else return false;
}
template <class F>
constexpr int local_out_cap(int lo, int hi, int t) {
  if constexpr (HasLocalRec<F>::value) return F::local_out_cap(lo, hi, t);
  else return 0;
}
template <class F, bool kHas = HasLocalRec<F>::value>
struct LocalRec {
  template <int SS, int LO, int HI, class C>
  static __device__ __forceinline__ void run(C&, const uint8_t*, int) {}
};
template <class F>
struct LocalRec<F, true> {
  template <int SS, int LO, int HI, class C>
  static __device__ __forceinline__ void run(C& ctx, const uint8_t* items, int n) {
    F::template exec_local<SS, LO, HI>(ctx, items, n);
  }
};

// A family may let the worker warps of a kernel [lo, hi] publish their ring outputs
// themselves (F::direct_publish(lo, hi, rtc), through Ctx::publish_warp): the kernel then
// has no block out buffers and runs as a sink group (no publisher warp, no round
// barrier), so warps that finish their share of a batch go on to the next one.
// F::direct_out_cap(lo, hi, t) is what one block can have in flight to t (ring sizing).
template <class F, class = void>
struct HasDirect : std::false_type {};
template <class F>
struct HasDirect<F, std::void_t<decltype(F::direct_publish(0, 0, false))>> : std::true_type {};
template <class F>
constexpr bool direct_publish(int lo, int hi, bool rtc) {
  if constexpr (HasDirect<F>::value) return F::direct_publish(lo, hi, rtc);
  else return false;
}
template <class F>
constexpr int direct_out_cap(int lo, int hi, bool rtc, int t) {
  if constexpr (HasDirect<F>::value) return F::direct_publish(lo, hi, rtc) ? F::direct_out_cap(lo, hi, t) : 0;
  else return 0;
}

// ------------------------------------------------------------------ constexpr graph helpers
template <class F>
struct Graph {
  static constexpr int S = F::S;
  static constexpr int fan(int s, int t) { return F::fanout(s, t); }
  // true iff an edge s->t with LO <= t <= s <= HI exists (recursion / loop inside [LO,HI])
  static constexpr bool has_back_edge(int lo, int hi) {
    for (int s = lo; s <= hi; ++s)
      for (int t = lo; t <= s; ++t)
        if (fan(s, t) > 0) return true;
    return false;
  }
  static constexpr bool rtc_legal(int lo, int hi) { return !has_back_edge(lo, hi) && F::rtc_ok(lo, hi); }
  static constexpr int mb(int lo, int hi, bool rtc, int s) { return kernel_max_batch<F>(lo, hi, rtc, s); }
  // items that can arrive block-locally at stage t of an RTC group [lo,hi]
  static constexpr int rtc_in_cap(int lo, int hi, int t) {
    if (t == lo) return mb(lo, hi, true, lo);
    int n = mb(lo, hi, true, t);
    int inc = 0;
    for (int s = lo; s < t; ++s) inc += rtc_in_cap(lo, hi, s) * fan(s, t);
    return n > inc ? n : inc;
  }
  // out-buffer capacity (items) for target t in a kernel [lo,hi]
  static constexpr int out_cap(int lo, int hi, bool rtc, int t) {
    if (direct_publish<F>(lo, hi, rtc)) return 0;  // no block out buffers
    if (rtc && lo < t && t <= hi && fused_chain<F>(lo, hi)) return fused_local_cap<F>(lo, hi, t);
    if (local_recursion<F>(lo, hi, rtc)) return local_out_cap<F>(lo, hi, t);
    int c = 0;
    for (int s = lo; s <= hi; ++s) {
      if (fan(s, t) == 0) continue;
      int n = rtc ? rtc_in_cap(lo, hi, s) : mb(lo, hi, false, s);
      int v = n * fan(s, t);
      if (rtc) c += v;
      else c = c > v ? c : v;
    }
    return c;
  }
  static constexpr int align128(int b) { return (b + 127) / 128 * 128; }
  static constexpr int in_region(int lo, int hi, bool rtc) {
    int b = 0;
    for (int s = lo; s <= hi; ++s) {
      int v = mb(lo, hi, rtc, s) * F::stride(s);
      b = b > v ? b : v;
    }
    return align128(b);
  }
  static constexpr int out_off(int lo, int hi, bool rtc, int t) {
    int off = 0;
    for (int u = 0; u < t; ++u) off += align128(out_cap(lo, hi, rtc, u) * F::stride(u));
    return off;
  }
  static constexpr int out_region(int lo, int hi, bool rtc) { return out_off(lo, hi, rtc, S); }
  // double-buffered: in[2] | out[2] | scratch
  static constexpr int in_base(int lo, int hi, bool rtc, int b) { return b * in_region(lo, hi, rtc); }
  static constexpr int out_base(int lo, int hi, bool rtc, int b) { return 2 * in_region(lo, hi, rtc) + b * out_region(lo, hi, rtc); }
  static constexpr int scratch_offset(int lo, int hi, bool rtc) { return out_base(lo, hi, rtc, 2); }
  // Block-local queues ("distributed queues"): in a
  // persistent, non-RTC kernel every self-recursive stage t (t -> t) gets a single-producer
  // (publisher warp) single-consumer (fetcher warp) ring in shared memory; children of t
  // stay in the producing block up to one batch, the rest goes to the global ring.
  static constexpr int pow2ceil(int v) {
    int p = 1;
    while (p < v) p <<= 1;
    return p;
  }
  // one default batch per queue (a larger configured batch just keeps fewer children
  // local); none at all if the queues would cost the kernel a resident block per SM
  // (shared memory: 228 KB per SM, ~1 KB reserved + ~2 KB static per block)
  static constexpr int lq_want(int lo, int hi, bool rtc, int t) {
    return (!rtc && !local_recursion<F>(lo, hi, rtc) && !direct_publish<F>(lo, hi, rtc) && lo <= t && t <= hi &&
            fan(t, t) > 0)
               ? pow2ceil(F::default_batch(t) < mb(lo, hi, false, t) ? F::default_batch(t) : mb(lo, hi, false, t))
               : 0;
  }
  static constexpr int smem_blocks(int dyn) { return (228 * 1024) / (dyn + 3 * 1024); }
  static constexpr bool lq_fits(int lo, int hi, bool rtc) {
    const int base = scratch_offset(lo, hi, rtc) + scratch_of<F>(lo, hi, rtc);
    int b = align128(base);
    for (int u = 0; u < S; ++u) b += align128(lq_want(lo, hi, rtc, u) * F::stride(u));
    return b <= 224 * 1024 && smem_blocks(b) >= smem_blocks(base);
  }
  static constexpr int lq_cap(int lo, int hi, bool rtc, int t) { return lq_fits(lo, hi, rtc) ? lq_want(lo, hi, rtc, t) : 0; }
  static constexpr int lq_off(int lo, int hi, bool rtc, int t) {
    int off = align128(scratch_offset(lo, hi, rtc) + scratch_of<F>(lo, hi, rtc));
    for (int u = 0; u < t; ++u) off += align128(lq_cap(lo, hi, rtc, u) * F::stride(u));
    return off;
  }
  static constexpr bool any_lq(int lo, int hi, bool rtc) {
    for (int t = 0; t < S; ++t)
      if (lq_cap(lo, hi, rtc, t) > 0) return true;
    return false;
  }
  static constexpr int smem_bytes(int lo, int hi, bool rtc) {
    return any_lq(lo, hi, rtc) ? lq_off(lo, hi, rtc, S) : scratch_offset(lo, hi, rtc) + scratch_of<F>(lo, hi, rtc);
  }
};

// ------------------------------------------------------------------ per-block context
struct BlockShared {
  int out_cnt[2][kMaxStages];          // per out buffer, per target
  unsigned long long out_base[kMaxStages];
  int nx_stage, nx_n, nx_seed, done;   // the batch the fetcher staged for the next round
  unsigned long long nx_base;
  long long acc_neg;                   // completions not yet subtracted from `pending` (<= 0)
  long long wave_rem;                  // WAVE: items of this block's chunk not yet claimed
  unsigned long long idle_since;       // %globaltimer when the fetcher last started idling (0: busy)
  unsigned long long deq[kMaxStages];
  unsigned long long enq[kMaxStages];
  uint32_t units32[kMaxStages];        // family-defined work units (Ctx::note_units)
  uint32_t deq32[kMaxStages], enq32[kMaxStages];  // counts added by several warps at once (native
                                                  // 32-bit shared atomics; 64-bit ones are CAS loops)
  unsigned long long t_exec[kMaxStages], t_flush[kMaxStages], t_idle, rounds;
  unsigned long long mbar[2];          // bulk-copy completion, one per in buffer
  uint32_t mbar_phase[2];
  int work[2];                         // per in buffer work counter (dynamic hand-out within a batch)
  // sink groups (no ring outputs): buffer hand-over without the round barrier
  unsigned long long full[2], empty[2];  // mbarriers: fetcher -> workers, workers -> fetcher
  int bn[2], bstage[2];                // items (-1: stop) and stage of each in buffer
  int lq_head[kMaxStages], lq_tail[kMaxStages];  // block-local queues (publisher -> fetcher)
  // cluster work stealing (F::kClusterSteal, cluster launch): the consumer side of each
  // block-local queue is taken under lq_lock by the owner's fetcher or the sibling's
  int lq_lock[kMaxStages];
  int steal_s;                         // stage of the batch being consumed under a lock (-1 none)
  uint32_t stolen32[kMaxStages];       // items this block took from its sibling's queues
  int alive;                           // admitted (the sibling may steal from this block)
  int sib_alive;                       // the cluster sibling was admitted (steals from it allowed)
  int steal_on;                        // this launch steals (Runner::steal_active)
};

// queue helpers defined below, used by Ctx::publish_warp
__device__ __forceinline__ void wait_slots(const Common& c, const QueueDesc& q, unsigned long long base, int n,
                                           int mode, int lane);
template <int STRIDE>
__device__ __forceinline__ void copy_out(uint8_t* ring, const uint8_t* src, unsigned long long base, int n,
                                         uint32_t cap_log2, int lane);

__device__ __forceinline__ void worker_sync() { asm volatile("bar.sync 1, %0;" ::"n"(kThreads) : "memory"); }

template <class F, int LO, int HI, bool RTC>
struct Ctx {
  using G = Graph<F>;
  const KArgs<F>& a;
  uint8_t* smem;
  BlockShared& sh;
  int ob;  // current out buffer

  __device__ Ctx(const KArgs<F>& a_, uint8_t* smem_, BlockShared& sh_) : a(a_), smem(smem_), sh(sh_), ob(0) {}
  static constexpr int kLo = LO, kHi = HI;  // the kernel's stage range (per-kernel code choices)
  static constexpr bool kRtc = RTC;

  __device__ __forceinline__ const typename F::Params& params() const { return a.p; }
  // layout constants are forced to compile time (nvcc does not always fold the
  // recursive constexpr helpers when they appear in runtime expressions)
  static constexpr int kScratch = G::scratch_offset(LO, HI, RTC);
  static constexpr int kOutBase0 = G::out_base(LO, HI, RTC, 0);
  static constexpr int kOutRegion = G::out_region(LO, HI, RTC);
  template <int T>
  struct OutT {
    static constexpr int off = G::out_off(LO, HI, RTC, T);
    static constexpr int cap = G::out_cap(LO, HI, RTC, T);
  };

  __device__ __forceinline__ uint8_t* scratch() { return smem + kScratch; }
  // Zero at the start of every round: worker warps may hand out the batch's items among
  // themselves with atomicAdd on it (dynamic load balance inside a batch).
  __device__ __forceinline__ int* work_counter() { return &sh.work[ob]; }

  template <int T>
  __device__ __forceinline__ uint8_t* out_ptr(int slot) {
    return smem + kOutBase0 + ob * kOutRegion + OutT<T>::off + slot * F::stride(T);
  }
  template <int T>
  static constexpr int cap() { return OutT<T>::cap; }
  // out slot of target T in out buffer b (either buffer, independent of the current one)
  template <int T>
  __device__ __forceinline__ uint8_t* out_ptr_in(int b, int slot) {
    return smem + kOutBase0 + b * kOutRegion + OutT<T>::off + slot * F::stride(T);
  }

  // Reserve k consecutive out slots for target T (one thread).  The declared fan-out
  // bounds guarantee capacity; exceeding it aborts the run (ABORT_FANOUT).
  template <int T>
  __device__ __forceinline__ int reserve(int k = 1) {
    int slot = atomicAdd(&sh.out_cnt[ob][T], k);
    if (slot + k > cap<T>()) {
      atomicCAS((unsigned long long*)&a.c.ctrl->abort.v, 0ull, (unsigned long long)ABORT_FANOUT);
      return -1;
    }
    return slot;
  }
  // A fused RTC chain executed n block-local items of stage T: the per-stage task count
  // (one thread per chain call).
  template <int T>
  __device__ __forceinline__ void note_local_count(int n) {
    sh.deq[T] += (unsigned long long)n;
    sh.enq[T] += (unsigned long long)n;  // entered stage T block-locally (sum enq == sum deq holds)
  }
  // As note_local_count, from any number of threads at once (direct-publish kernels,
  // whose warps run independently).
  template <int T>
  __device__ __forceinline__ void note_local_count_atomic(int n) {
    if (n) {
      atomicAdd(&sh.deq32[T], (uint32_t)n);
      atomicAdd(&sh.enq32[T], (uint32_t)n);
    }
  }
  // Warp-cooperative enqueue<T> of n <= 32 items staged contiguously in shared memory,
  // straight from a worker warp (direct-publish kernels; same protocol as the publisher
  // warp's: children counted in `pending` before they are visible, tail reservation,
  // free-slot wait, 16-B .cg payload stores, one release fence, per-slot sequence release,
  // `count` add).  All 32 lanes call it with the same arguments.
  template <int T>
  __device__ void publish_warp(const uint8_t* items, int n) {
    const int lane = threadIdx.x & 31;
    Ctrl* c = a.c.ctrl;
    const QueueDesc& q = a.c.q[T];
    unsigned long long base = 0;
    if (lane == 0) {
      red_add(&c->pending.v, n);
      if (a.g.group >= 0) {
        const int tg = a.c.stage_group[T];
        if (tg >= 0) red_add(&c->gpend[tg].v, n);
      }
      base = atom_add(&c->tail[T].v, n);
      atomicAdd(&sh.enq32[T], (uint32_t)n);
      if (a.c.flags & FLAG_DEPTH) {
        const unsigned long long h = ld_relaxed(&c->head[T].v);
        const unsigned long long dd = base + n - h;
        if (dd > c->max_depth[T]) atomicMax(&c->max_depth[T], dd);
      }
    }
    base = __shfl_sync(0xffffffffu, base, 0);
    const unsigned long long mask = (1ull << q.cap_log2) - 1;
    bool ok = true;
    for (int k = lane; k < n; k += 32) ok &= ld_acquire(q.seq + ((base + k) & mask)) == base + k;
    if (!__all_sync(0xffffffffu, ok)) wait_slots(a.c, q, base, n, 1, lane);
    __syncwarp();
    copy_out<F::stride(T)>(q.slots, items, base, n, q.cap_log2, lane);
    __syncwarp();
    fence_acq_rel_gpu();
    for (int k = lane; k < n; k += 32) st_relaxed(q.seq + ((base + k) & mask), base + k + 1);
    __syncwarp();
    if (lane == 0) red_add(&c->count[T].v, n);
  }
  // ... and, with FLAG_TRACE, the trace record of one of them (one thread per item).
  template <int T>
  __device__ __forceinline__ void trace_local(const uint8_t* item) {
    if (a.c.flags & FLAG_TRACE) {
      unsigned long long idx = atomicAdd(&a.c.ctrl->trace_n.v, 1ull);
      if (idx < a.c.trace_cap) {
        a.c.trace[idx].id = F::template item_id<T>(item);
        a.c.trace[idx].stage = T;
        a.c.trace[idx].smid = smid();
        a.c.trace[idx].kslot = (uint32_t)a.g.kslot;
        a.c.trace[idx].block = blockIdx.x;
      }
    }
  }
  // Family-defined work units of stage T (vp_run_stats.work_units; e.g. Reyes: the
  // micropolygons Shade actually shades), from any number of threads at once.
  template <int T>
  __device__ __forceinline__ void note_units(int n) {
    if (n) atomicAdd(&sh.units32[T], (uint32_t)n);
  }
  __device__ __forceinline__ bool tracing() const { return (a.c.flags & FLAG_TRACE) != 0; }
  // ... or given the task's item id directly (items that live only in registers).
  template <int T>
  __device__ __forceinline__ void trace_local_id(unsigned long long id) {
    if (a.c.flags & FLAG_TRACE) {
      unsigned long long idx = atomicAdd(&a.c.ctrl->trace_n.v, 1ull);
      if (idx < a.c.trace_cap) {
        a.c.trace[idx].id = id;
        a.c.trace[idx].stage = T;
        a.c.trace[idx].smid = smid();
        a.c.trace[idx].kslot = (uint32_t)a.g.kslot;
        a.c.trace[idx].block = blockIdx.x;
      }
    }
  }
  // Thread-level emit of a whole item (enqueue<Stage>(itemVal), Fig. 9 L37).
  template <int T>
  __device__ __forceinline__ void emit(const void* item) {
    int slot = reserve<T>();
    if (slot < 0) return;
    constexpr int W = F::stride(T) / 4;
    const uint32_t* src = (const uint32_t*)item;
    uint32_t* dst = (uint32_t*)out_ptr<T>(slot);
#pragma unroll
    for (int i = 0; i < W; ++i) dst[i] = src[i];
  }
  __device__ __forceinline__ void abort(unsigned long long why) {
    atomicCAS((unsigned long long*)&a.c.ctrl->abort.v, 0ull, why);
  }
};

// ------------------------------------------------------------------ queue operations
__device__ __forceinline__ bool aborted(const Ctrl* c) {
  return *(volatile const unsigned long long*)&c->abort.v != 0ull;
}

// Non-concurrent scheduling (a profiler serialising kernels, MPS, a co-tenant): CUDA does
// not guarantee that separately launched grids run concurrently, and a coarse/fine/hybrid
// plan needs every group resident.  A block that has been stalled for kCoresidentNs checks
// whether some planned kernel still has no block that ran its prologue; if so the run
// aborts (the host reruns it as one cooperative megakernel, vp_run_stats.model_rerun).
__device__ __forceinline__ bool peers_missing(const Common& c) {
  for (uint32_t m = c.peer_mask; m; m &= m - 1) {
    const int k = __ffs(m) - 1;
    if (ld_relaxed(&c.ctrl->arrivals[k].v) == 0ull) return true;
  }
  return false;
}
__device__ __forceinline__ bool check_coresident(const Common& c, unsigned long long stalled_ns) {
  if (stalled_ns < kCoresidentNs || !c.peer_mask || !peers_missing(c)) return false;
  if (atomicCAS((unsigned long long*)&c.ctrl->abort.v, 0ull, (unsigned long long)ABORT_NOT_CORESIDENT) == 0ull &&
      c.host_arrive) {
    // tell the host thread, which may be waiting for a grid that cannot be dispatched
    c.host_arrive[kMaxKernels] = c.epoch;
    __threadfence_system();
  }
  return true;
}

// One thread: claim up to k published items of stage s from its ring.
// 2 L2 atomics per block batch: `count` (availability) then `head` (ticket range).
__device__ __forceinline__ int claim_ring(Ctrl* c, int s, int k, unsigned long long& base) {
  long long avail = (long long)ld_relaxed(&c->count[s].v);
  if (avail <= 0) return 0;  // cheap L2 read first: idle fetchers do not hammer atomics
  int want = (int)(avail < k ? avail : k);
  long long old = (long long)atom_add(&c->count[s].v, -want);
  int got = old <= 0 ? 0 : (old < want ? (int)old : want);
  if (got < want) atom_add(&c->count[s].v, want - got);
  if (got == 0) return 0;
  base = atom_add(&c->head[s].v, got);
  return got;
}
// As claim_ring, with `avail` already polled (the fetcher polls all stages at once).
__device__ __forceinline__ int claim_ring_avail(Ctrl* c, int s, int k, long long avail, unsigned long long& base) {
  int want = (int)(avail < k ? avail : k);
  long long old = (long long)atom_add(&c->count[s].v, -want);
  int got = old <= 0 ? 0 : (old < want ? (int)old : want);
  if (got < want) atom_add(&c->count[s].v, want - got);
  if (got == 0) return 0;
  base = atom_add(&c->head[s].v, got);
  return got;
}
// One thread: claim up to k seed items of stage s.
__device__ __forceinline__ int claim_seed(Ctrl* c, const QueueDesc& q, int s, int k, unsigned long long& base) {
  if (q.n_seeds == 0) return 0;
  if ((long long)ld_relaxed(&c->seed_head[s].v) >= q.n_seeds) return 0;
  long long old = (long long)atom_add(&c->seed_head[s].v, k);
  if (old >= q.n_seeds) return 0;
  long long got = q.n_seeds - old;
  base = (unsigned long long)old;
  return (int)(got < k ? got : k);
}

// Warp-wide (lane = 0..31): wait until ring slots [base, base+n) hold the wanted sequence.
// mode 0: wait for publish (seq == t+1); mode 1: wait for free (seq == t).
__device__ __forceinline__ void wait_slots(const Common& c, const QueueDesc& q, unsigned long long base, int n,
                                           int mode, int lane) {
  const unsigned long long mask = (1ull << q.cap_log2) - 1;
  for (int k = lane; k < n; k += 32) {
    unsigned long long t = base + k;
    unsigned long long want = t + (mode == 0 ? 1ull : 0ull);
    const unsigned long long* p = q.seq + (t & mask);
    if (ld_acquire(p) == want) continue;
    unsigned long long t0 = globaltimer();
    unsigned ns = 32;
    while (ld_acquire(p) != want) {
      __nanosleep(ns);
      if (ns < 1024) ns <<= 1;
      if (aborted(c.ctrl)) return;
      unsigned long long now = globaltimer();
      if (mode == 1 && check_coresident(c, now - t0)) return;  // the consumer group never started
      // a producer stuck > 200 ms on a full ring is a capacity failure, not progress
      if (mode == 1 && now - t0 > 200000000ull) {
        atomicCAS((unsigned long long*)&c.ctrl->abort.v, 0ull, (unsigned long long)ABORT_OVERFLOW);
        return;
      }
      if (now > c.ctrl->deadline.v) {
        atomicCAS((unsigned long long*)&c.ctrl->abort.v, 0ull, (unsigned long long)ABORT_TIMEOUT);
        return;
      }
    }
  }
}

// Warp-wide copies between a smem batch and a ring (wrap-aware) or the seed array, in
// 16-B (or 8/4-B for small items) chunks, 4 loads in flight per lane; ring loads bypass
// L1 (.cg) so a reused slot is never served stale.
template <int STRIDE>
__device__ __forceinline__ void copy_in(uint8_t* dst, const uint8_t* ring, unsigned long long base, int n,
                                        uint32_t cap_log2, int lane) {
  using C = Chunk<STRIDE>;
  using T = typename C::T;
  const unsigned long long mask = (1ull << cap_log2) - 1;
  const int total = n * C::per_item;
  int i = lane;
  for (; i + 96 < total; i += 128) {
    T v[4];
#pragma unroll
    for (int u = 0; u < 4; ++u) {
      int j = i + 32 * u, k = j / C::per_item, w = j - k * C::per_item;
      v[u] = ld_cg((const T*)(ring + ((base + k) & mask) * STRIDE) + w);
    }
#pragma unroll
    for (int u = 0; u < 4; ++u) ((T*)dst)[i + 32 * u] = v[u];
  }
  for (; i < total; i += 32) {
    int k = i / C::per_item, w = i - k * C::per_item;
    ((T*)dst)[i] = ld_cg((const T*)(ring + ((base + k) & mask) * STRIDE) + w);
  }
}
template <int STRIDE>
__device__ __forceinline__ void copy_seed_in(uint8_t* dst, const uint8_t* seeds, unsigned long long base, int n,
                                             int lane) {
  using C = Chunk<STRIDE>;
  using T = typename C::T;
  const T* src = (const T*)(seeds + base * STRIDE);
  const int total = n * C::per_item;
  int i = lane;
  for (; i + 96 < total; i += 128) {
    T v[4];
#pragma unroll
    for (int u = 0; u < 4; ++u) v[u] = __ldg(src + i + 32 * u);
#pragma unroll
    for (int u = 0; u < 4; ++u) ((T*)dst)[i + 32 * u] = v[u];
  }
  for (; i < total; i += 32) ((T*)dst)[i] = __ldg(src + i);
}
template <int STRIDE>
__device__ __forceinline__ void copy_out(uint8_t* ring, const uint8_t* src, unsigned long long base, int n,
                                         uint32_t cap_log2, int lane) {
  using C = Chunk<STRIDE>;
  using T = typename C::T;
  const unsigned long long mask = (1ull << cap_log2) - 1;
  const int total = n * C::per_item;
  for (int i = lane; i < total; i += 32) {
    int k = i / C::per_item, w = i - k * C::per_item;
    st_cg((T*)(ring + ((base + k) & mask) * STRIDE) + w, ((const T*)src)[i]);
  }
}

// One thread: bulk copies of ring tickets [base, base+n) <-> a contiguous smem batch.
template <int STRIDE>
__device__ __forceinline__ void bulk_in(uint8_t* dst, const uint8_t* ring, unsigned long long base, int n,
                                        uint32_t cap_log2, unsigned long long* m) {
  const unsigned long long cap = 1ull << cap_log2, i0 = base & (cap - 1);
  const int n1 = (cap - i0) < (unsigned long long)n ? (int)(cap - i0) : n;
  mbar_arrive_expect_tx(m, (uint32_t)(n * STRIDE));
  bulk_g2s(dst, ring + i0 * STRIDE, (uint32_t)(n1 * STRIDE), m);
  if (n1 < n) bulk_g2s(dst + n1 * STRIDE, ring, (uint32_t)((n - n1) * STRIDE), m);
}
template <int STRIDE>
__device__ __forceinline__ void bulk_out(uint8_t* ring, const uint8_t* src, unsigned long long base, int n,
                                         uint32_t cap_log2) {
  const unsigned long long cap = 1ull << cap_log2, i0 = base & (cap - 1);
  const int n1 = (cap - i0) < (unsigned long long)n ? (int)(cap - i0) : n;
  bulk_s2g(ring + i0 * STRIDE, src, (uint32_t)(n1 * STRIDE));
  if (n1 < n) bulk_s2g(ring, src + n1 * STRIDE, (uint32_t)((n - n1) * STRIDE));
}

// ------------------------------------------------------------------ compile-time loops
template <int I, int N, class Fn>
__device__ __forceinline__ void static_for(Fn&& fn) {
  if constexpr (I < N) {
    fn(std::integral_constant<int, I>{});
    static_for<I + 1, N>(fn);
  }
}

// ------------------------------------------------------------------ the persistent block
// Warp-specialised persistent block (B200 design): warps 0..7 execute
// batch i of their stage, while the fetcher warp claims and stages batch i+1 and the
// publisher warp pushes the outputs of batch i-1 — the task scheduler and work-queue
// library of Fig. 2/Fig. 8 run concurrently with the stage functions, one block
// barrier per batch.
template <class F, int LO, int HI, bool RTC>
struct Runner {
  using G = Graph<F>;
  using CtxT = Ctx<F, LO, HI, RTC>;
  static constexpr int S = F::S;
  static constexpr int W_FETCH = kWarpsW, W_PUBLISH = kWarpsW + 1;
  static constexpr bool kSteal = HasClusterSteal<F>::value && !RTC && G::any_lq(LO, HI, RTC);
  // this launch steals: a persistent kernel with the flag, launched as clusters of 2
  static __device__ __forceinline__ bool steal_active(const KArgs<F>& a) {
    return kSteal && (a.c.flags & FLAG_STEAL) && a.g.mode == MODE_PERSISTENT && cluster_nctarank() == 2;
  }

  static constexpr int kInRegion = G::in_region(LO, HI, RTC);
  __device__ static __forceinline__ uint8_t* in_buf(uint8_t* smem, int b) { return smem + b * kInRegion; }
  template <int T>
  __device__ static __forceinline__ uint8_t* out_buf(uint8_t* smem, int b) {
    return smem + CtxT::kOutBase0 + b * CtxT::kOutRegion + CtxT::template OutT<T>::off;
  }

  template <int T>
  static constexpr int kLQ = G::lq_cap(LO, HI, RTC, T);
  template <int T>
  __device__ static __forceinline__ uint8_t* lq_buf(uint8_t* smem) { return smem + G::lq_off(LO, HI, RTC, T); }
  // warp copy of n items between a contiguous smem batch and a block-local ring (wrap-aware)
  template <int T, bool kToRing>
  __device__ static __forceinline__ void lq_copy(uint8_t* smem, uint8_t* batch, int first, int n, int lane) {
    using V = typename Chunk<F::stride(T)>::T;  // 16-B vectors when the stride allows
    constexpr int W = Chunk<F::stride(T)>::per_item;
    V* q = (V*)lq_buf<T>(smem);
    V* b = (V*)batch;
    for (int i = lane; i < n * W; i += 32) {
      const int k = i / W, w = i - k * W;
      const int slot = (first + k) & (kLQ<T> - 1);
      if (kToRing) q[slot * W + w] = b[i];
      else b[i] = q[slot * W + w];
    }
  }

  // ---------------- publisher warp: push out buffer `pb` (outputs of a batch of
  // `completed` items of stage ps) to the target rings, then retire the batch.
  // Lane T handles target T's reservation, so every L2 round trip of a publish is taken
  // once for all targets: tail reservations (1), free-slot check (1), bulk payload
  // store + completion (1), sequence release.
  static __device__ void publish(const KArgs<F>& a, BlockShared& sh, uint8_t* smem, int pb, int ps, int completed,
                                 int lane) {
    Ctrl* c = a.c.ctrl;
    const bool timers = a.c.flags & FLAG_TIMERS;
    unsigned long long t0 = (timers && lane == 0) ? globaltimer() : 0;
    int myn = 0;  // lane T: items for target T (clamped to the declared capacity)
    static_for<0, S>([&](auto T_) {
      constexpr int T = decltype(T_)::value;
      constexpr int capT = CtxT::template cap<T>();
      if (lane == T) {
        const int n = sh.out_cnt[pb][T];
        myn = n > capT ? capT : n;
      }
    });
    int children = myn;
#pragma unroll
    for (int o = 16; o; o >>= 1) children += __shfl_xor_sync(0xffffffffu, children, o);
    if (children == 0) {
      if (lane == 0) {
        sh.acc_neg -= completed;
        if (timers) sh.t_flush[ps] += globaltimer() - t0;
      }
      return;
    }
    // Termination accounting: children are counted in `pending` before they become
    // visible (the release stores below order this reduction before them); completions
    // may be deferred (pending only stays conservatively high).
    // per-group alive counts (online adaptation): children into this kernel's own group and
    // its completions go in ONE atomic, so the group's count never dips to 0 transiently
    const int tg = (myn > 0) ? (int)a.c.stage_group[lane] : -1;
    int own = (tg >= 0 && tg == a.g.group) ? myn : 0;
#pragma unroll
    for (int o = 16; o; o >>= 1) own += __shfl_xor_sync(0xffffffffu, own, o);
    if (a.g.group >= 0) {
      // online adaptation: children counted in their target groups BEFORE this group's
      // completions are subtracted, so no observer can see this group drained (gpend 0)
      // while its children are not yet counted downstream (the target could otherwise
      // retire with items in its ring)
      if (tg >= 0 && tg != a.g.group) red_add(&c->gpend[tg].v, myn);
      __syncwarp();
      fence_acq_rel_gpu();
    }
    if (lane == 0) {
      const long long d = children - completed + sh.acc_neg;
      if (d != 0) red_add(&c->pending.v, d);
      const long long dg = own - completed + sh.acc_neg;
      if (a.g.group >= 0 && dg != 0) red_add(&c->gpend[a.g.group].v, dg);
      sh.acc_neg = 0;
    }
    // block-local queues first (self-recursive targets): lane T keeps up to one batch of
    // its children in the block, the rest (myg) goes to the global ring
    int myloc = 0;
    if (a.g.mode == MODE_PERSISTENT) {
      static_for<0, S>([&](auto T_) {
        constexpr int T = decltype(T_)::value;
        if constexpr (kLQ<T> > 0) {
          if (lane == T && myn > 0) {
            const int occ = sh.lq_tail[T] - *(volatile int*)&sh.lq_head[T];
            const int lim = a.g.batch[T] < kLQ<T> ? a.g.batch[T] : kLQ<T>;
            myloc = lim - occ < myn ? lim - occ : myn;
            if (myloc < 0) myloc = 0;
          }
          const int nl = __shfl_sync(0xffffffffu, myloc, T);
          if (nl > 0) {
            __threadfence_block();  // the consumer's reads of these slots came before its head update
            lq_copy<T, true>(smem, out_buf<T>(smem, pb), sh.lq_tail[T], nl, lane);
            __syncwarp();
            if (lane == T) {
              // items before the tail that publishes them (to the sibling too, when it may steal)
              if (kSteal && sh.steal_on) fence_acq_rel_cluster();
              else __threadfence_block();
              *(volatile int*)&sh.lq_tail[T] = sh.lq_tail[T] + nl;
            }
          }
        }
      });
    }
    if (myn > 0) sh.enq[lane] += myn;
    myn -= myloc;  // from here on: the items for the global ring, out buffer offset myloc
    unsigned long long mybase = 0;
    if (myn > 0) {
      mybase = atom_add(&c->tail[lane].v, myn);
      if (a.c.flags & FLAG_DEPTH) {
        const unsigned long long h = ld_relaxed(&c->head[lane].v);
        const unsigned long long dd = mybase + myn - h;
        if (dd > c->max_depth[lane]) atomicMax(&c->max_depth[lane], dd);
      }
    }
    // free-slot check: acquire loads of every target's slots (LDG + L1 invalidate, no
    // membar), all issued before any is tested
    bool free_ok = true;
    static_for<0, S>([&](auto T_) {
      constexpr int T = decltype(T_)::value;
      if constexpr (CtxT::template cap<T>() > 0) {
        const int n = __shfl_sync(0xffffffffu, myn, T);
        const unsigned long long base = __shfl_sync(0xffffffffu, mybase, T);
        const unsigned long long mask = (1ull << a.c.q[T].cap_log2) - 1;
        for (int k = lane; k < n; k += 32) free_ok &= ld_acquire(a.c.q[T].seq + ((base + k) & mask)) == base + k;
      }
    });
    if (!__all_sync(0xffffffffu, free_ok)) {
      // a consumer is still reading the previous lap of some slot (full ring): spin
      static_for<0, S>([&](auto T_) {
        constexpr int T = decltype(T_)::value;
        if constexpr (CtxT::template cap<T>() > 0) {
          const int n = __shfl_sync(0xffffffffu, myn, T);
          const unsigned long long base = __shfl_sync(0xffffffffu, mybase, T);
          if (n > 0) wait_slots(a.c, a.c.q[T], base, n, 1, lane);
        }
      });
    }
    __syncwarp();  // every slot of every range is free before any payload is written
    bool bulk_used = false;
    static_for<0, S>([&](auto T_) {
      constexpr int T = decltype(T_)::value;
      if constexpr (CtxT::template cap<T>() > 0) {
        const int n = __shfl_sync(0xffffffffu, myn, T);
        const unsigned long long base = __shfl_sync(0xffffffffu, mybase, T);
        if (n > 0) {
          const uint8_t* src = out_buf<T>(smem, pb) + (size_t)__shfl_sync(0xffffffffu, myloc, T) * F::stride(T);
          if constexpr (F::stride(T) % 16 == 0) {
            if (lane == 0) {
              fence_proxy_async_global();
              bulk_out<F::stride(T)>(a.c.q[T].slots, src, base, n, a.c.q[T].cap_log2);
            }
            bulk_used = true;
          } else {
            copy_out<F::stride(T)>(a.c.q[T].slots, src, base, n, a.c.q[T].cap_log2, lane);
          }
        }
      }
    });
    if (bulk_used && lane == 0) {
      bulk_commit_wait_all();       // payload written (and the smem batch read) ...
      fence_proxy_async_global();   // ... and ordered before the generic release below
    }
    __syncwarp();
    // publish: seq = ticket + 1.  One release fence for every target's sequence stores
    // (fence + relaxed stores = the release pattern; one membar per publish).
    fence_acq_rel_gpu();
    static_for<0, S>([&](auto T_) {
      constexpr int T = decltype(T_)::value;
      if constexpr (CtxT::template cap<T>() > 0) {
        const int n = __shfl_sync(0xffffffffu, myn, T);
        const unsigned long long base = __shfl_sync(0xffffffffu, mybase, T);
        const unsigned long long mask = (1ull << a.c.q[T].cap_log2) - 1;
        for (int k = lane; k < n; k += 32) st_relaxed(a.c.q[T].seq + ((base + k) & mask), base + k + 1);
      }
    });
    if (myn > 0) red_add(&c->count[lane].v, myn);
    if (lane < S) sh.out_cnt[pb][lane] = 0;
    if (timers && lane == 0) sh.t_flush[ps] += globaltimer() - t0;
  }

  // ---------------- fetcher warp: claim the next batch (task scheduler) and stage it
  // into in buffer nb.  quiescent: this block holds no batch and flushes nothing now.
  // Thief side of the cluster work stealing (fetcher lane 0): take up to half of the
  // sibling's block-local queue of the most downstream stage that has >= 2 items.  The
  // victim's consumer lock is held until the items are copied (fetch, nx_seed == 3).
  static __device__ __noinline__ int steal_claim(const KArgs<F>& a, BlockShared& sh, int& st, int& fs,
                                                 unsigned long long& base) {
    constexpr int NS = HI - LO + 1;
    const uint32_t sib = cluster_ctarank() ^ 1u;
    int got = 0;
    static_for<0, NS>([&](auto L_) {
      constexpr int l = decltype(L_)::value, s = HI - l;
      if constexpr (kLQ<s> > 0) {
        if (!got) {
          const uint32_t rh = dsmem_addr(&sh.lq_head[s], sib), rt = dsmem_addr(&sh.lq_tail[s], sib);
          if (dsmem_ld_relaxed(rt) - dsmem_ld_relaxed(rh) >= 2) {
            const uint32_t rl = dsmem_addr(&sh.lq_lock[s], sib);
            if (dsmem_trylock(rl)) {
              const int h = dsmem_ld_relaxed(rh), t = dsmem_ld_acquire(rt);
              const int k = min((t - h + 1) / 2, a.g.batch[s]);
              if (k > 0) {
                got = k;
                st = s;
                fs = 3;
                base = (unsigned long long)h;
                sh.steal_s = s;
              } else {
                dsmem_st_release(rl, 0);
              }
            }
          }
        }
      }
    });
    return got;
  }

  static __device__ void fetch(const KArgs<F>& a, BlockShared& sh, uint8_t* smem, int nb, bool quiescent, int lane) {
    Ctrl* c = a.c.ctrl;
    const bool timers = a.c.flags & FLAG_TIMERS;
    constexpr int NS = HI - LO + 1;
    // One warp-wide poll of every ring's `count` and seed cursor (one L2 round trip
    // instead of one per stage); lane l looks at stage HI - l (downstream first).
    long long avail = 0;
    bool seeds_left = false;
    if (a.g.mode != MODE_WAVE && lane < NS) {
      const int s = HI - lane;
      avail = (long long)ld_relaxed(&c->count[s].v);
      const long long ns = a.c.q[s].n_seeds;
      seeds_left = ns > 0 && (long long)ld_relaxed(&c->seed_head[s].v) < ns;
    }
    long long av[NS];
    static_for<0, NS>([&](auto L_) { av[decltype(L_)::value] = __shfl_sync(0xffffffffu, avail, decltype(L_)::value); });
    const unsigned seed_mask = __ballot_sync(0xffffffffu, seeds_left);
    if (lane == 0) {
      unsigned long long t0 = timers ? globaltimer() : 0;
      int got = 0, st = -1, fs = 0;
      unsigned long long base = 0;
      sh.done = 0;
      if (aborted(c)) {
        sh.done = 1;
      } else if (a.g.group >= 0 && *(volatile unsigned long long*)&c->retired[a.g.group]) {
        sh.done = 1;  // another block of this group retired it (nothing is left for it)
      } else if (globaltimer() > c->deadline.v) {
        // watchdog, checked every round even by busy blocks (the tuner's timeoutexec)
        atomicCAS((unsigned long long*)&c->abort.v, 0ull, (unsigned long long)ABORT_TIMEOUT);
        sh.done = 1;
      } else if (a.g.mode == MODE_WAVE) {
        const int s = a.g.wave_stage;
        int k = (int)(sh.wave_rem < a.g.batch[s] ? sh.wave_rem : a.g.batch[s]);
        if (k > 0) {
          got = claim_ring(c, s, k, base);
          fs = 0;
          if (!got) {
            got = claim_seed(c, a.c.q[s], s, k, base);
            fs = 1;
          }
          st = s;
          sh.wave_rem -= got;
          if (!got) sh.wave_rem = 0;  // cannot happen when the host sized the wave
        }
        if (!got && quiescent) sh.done = 1;
      } else {
        // "Query queues in turn of priority" (Fig. 8a): downstream stages first (drains
        // the pipeline, bounds live items), rings before seeds.
        static_for<0, NS>([&](auto L_) {
          constexpr int l = decltype(L_)::value, s = HI - l;
          if constexpr (kLQ<s> > 0) {  // this block's own children of s come first
            if (!got) {
              int occ = *(volatile int*)&sh.lq_tail[s] - sh.lq_head[s];
              if constexpr (kSteal) {
                // the consumer side is shared with the sibling: take it under the lock
                // and re-read head (a thief may have advanced it)
                if (occ > 0 && sh.steal_on) {
                  if (dsmem_trylock(dsmem_addr(&sh.lq_lock[s], cluster_ctarank()))) {
                    occ = *(volatile int*)&sh.lq_tail[s] - *(volatile int*)&sh.lq_head[s];
                    if (occ > 0) sh.steal_s = s;
                    else dsmem_st_release(dsmem_addr(&sh.lq_lock[s], cluster_ctarank()), 0);
                  } else {
                    occ = 0;  // a thief is copying from it; try the rings
                  }
                }
              }
              if (occ > 0) {
                got = occ < a.g.batch[s] ? occ : a.g.batch[s];
                st = s;
                fs = 2;
                base = (unsigned long long)(kSteal ? *(volatile int*)&sh.lq_head[s] : sh.lq_head[s]);
              }
            }
          }
          if (!got && av[l] > 0) {
            got = claim_ring_avail(c, s, a.g.batch[s], av[l], base);
            if (got) { st = s; fs = 0; }
          }
        });
        static_for<0, NS>([&](auto L_) {
          constexpr int l = decltype(L_)::value, s = HI - l;
          if (!got && ((seed_mask >> l) & 1u)) {
            got = claim_seed(c, a.c.q[s], s, a.g.batch[s], base);
            if (got) { st = s; fs = 1; }
          }
        });
        if constexpr (kSteal) {
          // nothing in this block's queues, the rings or the seeds: take up to half of the
          // cluster sibling's block-local queue over DSMEM (a separate, non-inlined path:
          // the plain fetch stays as it was)
          if (!got && sh.steal_on && sh.sib_alive) got = steal_claim(a, sh, st, fs, base);
        }
        if (!got && quiescent) {
          // idle: retire deferred completions first, then test for termination
          if (sh.acc_neg != 0) {
            atom_add(&c->pending.v, sh.acc_neg);
            if (a.g.group >= 0) atom_add(&c->gpend[a.g.group].v, sh.acc_neg);
            sh.acc_neg = 0;
          }
          if ((long long)ld_acquire(&c->pending.v) <= 0) {
            sh.done = 1;
          } else if (a.g.can_retire && group_drained(a)) {
            // nothing can reach this group's stages any more: retire it (its SMs go to
            // another group, the host launches the refill)
            atomicExch(&c->retired[a.g.group], 1ull);
            sh.done = 1;
          } else if (globaltimer() > c->deadline.v) {
            atomicCAS((unsigned long long*)&c->abort.v, 0ull, (unsigned long long)ABORT_TIMEOUT);
            sh.done = 1;
          } else {
            const unsigned long long now = globaltimer();
            if (!sh.idle_since) sh.idle_since = now;
            if (check_coresident(a.c, now - sh.idle_since)) sh.done = 1;
            else __nanosleep(256);
          }
        }
      }
      if (got) sh.idle_since = 0;
      sh.nx_stage = st;
      sh.nx_n = got;
      sh.nx_base = base;
      sh.nx_seed = fs;
      if (timers && !got) sh.t_idle += globaltimer() - t0;
    }
    __syncwarp();
    const int n = sh.nx_n;
    if (n == 0) return;
    const int s = sh.nx_stage;
    const unsigned long long base = sh.nx_base;
    uint8_t* dst = in_buf(smem, nb);
    unsigned long long* mb = &sh.mbar[nb];
    static_for<LO, HI + 1>([&](auto S_) {
      constexpr int SS = decltype(S_)::value;
      constexpr bool kBulk = F::stride(SS) % 16 == 0;
      if (s == SS) {
        const QueueDesc& q = a.c.q[SS];
        if (kBulk) fence_proxy_async_smem();  // earlier generic writes of this buffer -> bulk writes
        if (kLQ<SS> > 0 && sh.nx_seed == 2) {  // from the block-local queue
          if constexpr (kLQ<SS> > 0) {
            __threadfence_block();  // the items the observed tail published
            lq_copy<SS, false>(smem, dst, (int)base, n, lane);
            __syncwarp();
            if (lane == 0) {
              __threadfence_block();  // reads of the slots before the head frees them
              *(volatile int*)&sh.lq_head[SS] = (int)base + n;
              if constexpr (kSteal) {
                if (sh.steal_s >= 0) {  // taken under the queue's lock
                  dsmem_st_release(dsmem_addr(&sh.lq_lock[SS], cluster_ctarank()), 0);
                  sh.steal_s = -1;
                }
              }
            }
          }
        } else if (kSteal && kLQ<SS> > 0 && sh.nx_seed == 3) {  // from the sibling's queue
          if constexpr (kSteal && kLQ<SS> > 0) {
            using V = typename Chunk<F::stride(SS)>::T;
            constexpr int W = Chunk<F::stride(SS)>::per_item;
            const uint32_t sib = cluster_ctarank() ^ 1u;
            const uint32_t rq = dsmem_addr(lq_buf<SS>(smem), sib);  // same offset in the sibling
            V* bdst = (V*)dst;
            for (int i = lane; i < n * W; i += 32) {
              const int k = i / W, w = i - k * W;
              const int slot = ((int)base + k) & (kLQ<SS> - 1);
              bdst[i] = dsmem_ld<V>(rq + (uint32_t)((slot * W + w) * (int)sizeof(V)));
            }
            __syncwarp();
            if (lane == 0) {
              // the slots are read before the head that frees them, then the lock
              dsmem_st_release(dsmem_addr(&sh.lq_head[SS], sib), (int)base + n);
              dsmem_st_release(dsmem_addr(&sh.lq_lock[SS], sib), 0);
              sh.steal_s = -1;
              sh.stolen32[SS] += (uint32_t)n;
            }
          }
        } else if (sh.nx_seed) {
          if constexpr (kBulk) {
            if (lane == 0) {
              mbar_arrive_expect_tx(mb, (uint32_t)(n * F::stride(SS)));
              bulk_g2s(dst, q.seeds + base * F::stride(SS), (uint32_t)(n * F::stride(SS)), mb);
              mbar_wait(mb, sh.mbar_phase[nb]);
              sh.mbar_phase[nb] ^= 1u;
            }
          } else {
            copy_seed_in<F::stride(SS)>(dst, q.seeds, base, n, lane);
          }
        } else {
          // published? acquire loads (no membar); spin only if a producer lags
          const unsigned long long mask = (1ull << q.cap_log2) - 1;
          bool ok = true;
          for (int k = lane; k < n; k += 32) ok &= ld_acquire(q.seq + ((base + k) & mask)) == base + k + 1;
          if (!__all_sync(0xffffffffu, ok)) wait_slots(a.c, q, base, n, 0, lane);
          __syncwarp();
          // warp-uniform decision (lanes may observe the abort flag at different times)
          const bool abort_now = __shfl_sync(0xffffffffu, aborted(a.c.ctrl) ? 1 : 0, 0) != 0;
          if (abort_now) {  // never hand unpublished slots to the workers
            if (lane == 0) {
              sh.nx_n = 0;
              sh.done = 1;
            }
            return;
          }
          if constexpr (kBulk) {
            if (lane == 0) {
              fence_proxy_async_global();  // acquired payload -> async-proxy reads
              bulk_in<F::stride(SS)>(dst, q.slots, base, n, q.cap_log2, mb);
              mbar_wait(mb, sh.mbar_phase[nb]);  // bytes landed: the slots' reads are done
              sh.mbar_phase[nb] ^= 1u;
            }
          } else {
            copy_in<F::stride(SS)>(dst, q.slots, base, n, q.cap_log2, lane);
          }
          __syncwarp();
          fence_acq_rel_gpu();  // the batch's reads before the slots' release (one membar)
          for (int k = lane; k < n; k += 32) {
            unsigned long long t = base + k;
            st_relaxed(q.seq + (t & mask), t + (1ull << q.cap_log2));  // free for ticket t + cap
          }
        }
      }
    });
  }

  static __device__ __forceinline__ void record_trace(const KArgs<F>& a, int s, const uint8_t* items, int n) {
    if (!(a.c.flags & FLAG_TRACE)) return;
    uint32_t sm = smid();
    static_for<LO, HI + 1>([&](auto S_) {
      constexpr int SS = decltype(S_)::value;
      if (s == SS) {
        for (int k = threadIdx.x; k < n; k += kThreads) {
          unsigned long long idx = atomicAdd(&a.c.ctrl->trace_n.v, 1ull);
          if (idx < a.c.trace_cap) {
            a.c.trace[idx].id = F::template item_id<SS>(items + k * F::stride(SS));
            a.c.trace[idx].stage = SS;
            a.c.trace[idx].smid = sm;
            a.c.trace[idx].kslot = (uint32_t)a.g.kslot;
            a.c.trace[idx].block = blockIdx.x;
          }
        }
      }
    });
  }

  // ---------------- worker warps: execute stage s on n staged items into out buffer
  // ctx.ob; RTC groups then run the rest of the linear group on block-local items.
  static __device__ void execute(const KArgs<F>& a, CtxT& ctx, BlockShared& sh, int s, const uint8_t* items, int n) {
    const bool timers = a.c.flags & FLAG_TIMERS;
    unsigned long long t0 = (timers && threadIdx.x == 0) ? globaltimer() : 0;
    static_for<LO, HI + 1>([&](auto S_) {
      constexpr int SS = decltype(S_)::value;
      if (s == SS) {
        record_trace(a, SS, items, n);
        if (threadIdx.x == 0) atomicAdd(&sh.deq32[SS], (uint32_t)n);  // direct-publish warps add too
        // a fused chain runs in RTC kernels, and in local-recursion kernels (a megakernel
        // whose Bound / Split batches never use the out buffers) for the chain's stages
        if constexpr ((RTC || local_recursion<F>(LO, HI, RTC)) && SS < HI && fused_chain<F>(SS, HI)) {
          FusedChain<F>::template run<SS, HI>(ctx, items, n);
        } else if constexpr (local_recursion<F>(LO, HI, RTC)) {
          LocalRec<F>::template run<SS, LO, HI>(ctx, items, n);
        } else {
        F::template exec<SS>(ctx, items, n);
        if constexpr (RTC && SS < HI) {
          // RTC (L11 §4.1): the remaining stages of the linear group, block-locally.
          // Local items were never counted in `pending` (the claimed parents keep it
          // positive), so they are neither added nor retired.
          static_for<SS + 1, HI + 1>([&](auto T_) {
            constexpr int TT = decltype(T_)::value;
            worker_sync();
            int m = sh.out_cnt[ctx.ob][TT];
            constexpr int capT = CtxT::template cap<TT>();
            if (m > capT) m = capT;
            if (m > 0) {
              const uint8_t* loc = ctx.template out_ptr<TT>(0);
              record_trace(a, TT, loc, m);
              if (threadIdx.x == 0) sh.deq[TT] += m;
              F::template exec<TT>(ctx, loc, m);
            }
            worker_sync();
            if (threadIdx.x == 0) sh.out_cnt[ctx.ob][TT] = 0;  // consumed locally
          });
        }
        }
        fence_proxy_async_smem();  // out-buffer writes -> the publisher's bulk reads
        if (timers && threadIdx.x == 0) sh.t_exec[SS] += globaltimer() - t0;
      }
    });
  }

  static __device__ bool admit(const KArgs<F>& a, BlockShared& sh) {
    // check_sm() + check_sm_blk() (Fig. 5, L21; §5), increment-then-compare
    // (Fig. 5's check-then-increment is racy).
    __shared__ int ok;
    if (threadIdx.x == 0) {
      const GroupArgs& g = a.g;
      Ctrl* c = a.c.ctrl;
      int good = 1;
      uint32_t sm = smid();
      if (g.mode == MODE_PERSISTENT) {
        if (sm >= (uint32_t)kMaxSM || !((g.sm_mask[sm >> 5] >> (sm & 31)) & 1u)) good = 0;
        if (good && g.quota > 0) {
          uint32_t slot = atomicAdd(&a.c.blk[g.kslot * kMaxSM + sm], 1u);
          if (slot >= (uint32_t)g.quota) good = 0;
        } else if (good && sm < (uint32_t)kMaxSM) {
          atomicAdd(&a.c.blk[g.kslot * kMaxSM + sm], 1u);
        }
        if (good) atomicAdd(&c->admitted[g.kslot].v, 1ull);
        __threadfence();
        unsigned long long t = atomicAdd(&c->arrivals[g.kslot].v, 1ull);
        if (t == (unsigned long long)gridDim.x - 1 && a.c.host_arrive) {
          // every block of this grid has been dispatched and decided: the host may launch
          // the next group's kernel (deterministic SM/block binding)
          a.c.host_arrive[g.kslot] = a.c.epoch;
          __threadfence_system();
        }
        // progress guarantee: the last block of a grid to arrive stays if nobody did
        // (binding is a performance hint; correctness never depends on it)
        if (!good && t == (unsigned long long)gridDim.x - 1 && ld_relaxed(&c->admitted[g.kslot].v) == 0) {
          good = 1;
          atomicAdd(&c->admitted[g.kslot].v, 1ull);
          atomicAdd(&c->fallback_admits, 1ull);
        }
        // online adaptation: the grid's last block arrives after every admitted block of a
        // retired group already left -> it tells the host instead of them
        if (!good && t == (unsigned long long)gridDim.x - 1 && g.group >= 0 && a.c.host_retire &&
            *(volatile unsigned long long*)&c->retired[g.group] &&
            *(volatile unsigned long long*)&c->exits[g.kslot] == ld_relaxed(&c->admitted[g.kslot].v)) {
          signal_retired(a, g.kslot);
        }
      } else if (sm < (uint32_t)kMaxSM) {
        atomicAdd(&a.c.blk[g.kslot * kMaxSM + sm], 1u);
      }
      ok = good;
      for (int s = 0; s < kMaxStages; ++s) {
        sh.out_cnt[0][s] = sh.out_cnt[1][s] = 0;
        sh.deq[s] = sh.enq[s] = 0;
        sh.deq32[s] = sh.enq32[s] = sh.units32[s] = 0;
        sh.t_exec[s] = sh.t_flush[s] = 0;
      }
      sh.t_idle = 0;
      sh.rounds = 0;
      for (int b = 0; b < 2; ++b) {
        mbar_init(&sh.mbar[b], 1);
        sh.mbar_phase[b] = 0;
      }
      sh.acc_neg = 0;
      sh.idle_since = 0;
      sh.done = 0;
      sh.work[0] = sh.work[1] = 0;
      sh.nx_n = 0;
      sh.nx_stage = -1;
      for (int t = 0; t < kMaxStages; ++t) sh.lq_head[t] = sh.lq_tail[t] = 0;
      if constexpr (kSteal) {
        for (int t = 0; t < kMaxStages; ++t) {
          sh.lq_lock[t] = 0;
          sh.stolen32[t] = 0;
        }
        sh.steal_s = -1;
        sh.alive = 1;
        sh.sib_alive = 0;
      }
      sh.steal_on = steal_active(a) ? 1 : 0;
      if (g.mode == MODE_WAVE) {
        long long wn = g.wave_n, wc = g.wave_chunk;
        if (g.wave_n_dev) {
          // device-driven KBK (CUDA graph): the planner kernel sized this wave; split it
          // into whole batches over the fixed grid exactly like launch_wave does on the host
          wn = *g.wave_n_dev;
          const long long bt = g.batch[g.wave_stage];
          const long long batches = (wn + bt - 1) / bt;
          wc = ((batches + gridDim.x - 1) / gridDim.x) * bt;
          if (wc < bt) wc = bt;
        }
        long long lo = (long long)blockIdx.x * wc;
        long long rem = wn - lo;
        sh.wave_rem = rem < 0 ? 0 : (rem < wc ? rem : wc);
      } else {
        sh.wave_rem = 0;
      }
    }
    __syncthreads();
    return ok != 0;
  }

  // Tell the host that kernel k's SMs are free (online adaptation), with a snapshot of every
  // group's alive count so the host can give them to the group with the most stalled work.
  static __device__ void signal_retired(const KArgs<F>& a, int kslot) {
    if (a.c.host_gpend) {
      for (int g = 0; g < kMaxKernels; ++g)
        a.c.host_gpend[kslot * kMaxKernels + g] = (long long)ld_relaxed(&a.c.ctrl->gpend[g].v);
      __threadfence_system();
    }
    a.c.host_retire[kslot] = a.c.epoch;
    __threadfence_system();
  }

  static __device__ void flush_stats(const KArgs<F>& a, BlockShared& sh) {
    if (threadIdx.x == 0) {
      Ctrl* c = a.c.ctrl;
      if (sh.acc_neg != 0) atom_add(&c->pending.v, sh.acc_neg);
      if (sh.acc_neg != 0 && a.g.group >= 0) atom_add(&c->gpend[a.g.group].v, sh.acc_neg);
      sh.acc_neg = 0;
      for (int s = 0; s < S; ++s) {
        const unsigned long long dq = sh.deq[s] + sh.deq32[s], eq = sh.enq[s] + sh.enq32[s];
        if (dq) atomicAdd(&c->deq[s], dq);
        if (eq) atomicAdd(&c->enq[s], eq);
        if (sh.units32[s]) atomicAdd(&c->units[s], (unsigned long long)sh.units32[s]);
        if constexpr (kSteal) {
          if (sh.stolen32[s]) atomicAdd(&c->stolen[s], (unsigned long long)sh.stolen32[s]);
        }
        if (sh.t_exec[s]) atomicAdd(&c->exec_ns[s], sh.t_exec[s]);
        if (sh.t_flush[s]) atomicAdd(&c->flush_ns[s], sh.t_flush[s]);
      }
      if (sh.t_idle) atomicAdd(&c->idle_ns[a.g.kslot], sh.t_idle);
      atomicAdd(&c->rounds[a.g.kslot], sh.rounds);
      if (a.g.group >= 0 && a.c.host_retire && a.g.mode == MODE_PERSISTENT) {
        // the last admitted block of a retired group's kernel to leave tells the host
        // that the kernel's SMs are free (the grid is fully dispatched: every block that
        // will ever be admitted has been)
        __threadfence();
        const unsigned long long e = atomicAdd(&c->exits[a.g.kslot], 1ull) + 1;
        if (*(volatile unsigned long long*)&c->retired[a.g.group] &&
            ld_relaxed(&c->arrivals[a.g.kslot].v) == (unsigned long long)gridDim.x &&
            e == ld_relaxed(&c->admitted[a.g.kslot].v)) {
          signal_retired(a, a.g.kslot);
        }
      }
    }
  }

  // every feeder group retired and no item alive in this group's stages (seeds included)
  static __device__ __forceinline__ bool group_drained(const KArgs<F>& a) {
    Ctrl* c = a.c.ctrl;
    for (uint32_t f = a.g.feeders; f; f &= f - 1) {
      const int g = __ffs(f) - 1;
      if (!*(volatile unsigned long long*)&c->retired[g]) return false;
    }
    return (long long)ld_acquire(&c->gpend[a.g.group].v) <= 0;
  }

  // A sink group emits nothing to any ring (every successor of its stages is a later
  // stage of the same RTC chain, or none): it needs no publisher, so worker warps and the
  // fetcher hand the two in buffers over through mbarriers instead of a block barrier
  // per round.  A worker warp that finishes its share of batch i starts batch i+1 as
  // soon as the fetcher staged it, instead of waiting for the slowest warp of batch i.
  static constexpr bool no_ring_outputs() {
    for (int s = LO; s <= HI; ++s)
      for (int t = 0; t < S; ++t)
        if (F::fanout(s, t) > 0 && !(RTC && t > LO && t <= HI)) return false;
    return true;
  }
  // ... or its warps publish their outputs themselves (direct-publish kernels)
  static constexpr bool sink_group() { return direct_publish<F>(LO, HI, RTC) || no_ring_outputs(); }
  // A direct-publish kernel has no publisher warp at all: its blocks are the 8 worker
  // warps + the fetcher, so the register file is divided among 9 warps, not 10 (the
  // Reyes [Bound, Split] kernel: 56 registers at 4 blocks/SM, no spills; DESIGN.md
  // §4.3).  Measured A/B for the other sink groups (the fused [Dice, Shade] kernel):
  // 288 threads at 72 registers was 7% slower than 320 at 64, so they keep 320.
  static constexpr int kBlockThreads = direct_publish<F>(LO, HI, RTC) ? kThreads + 32 : kBlock;

  static __device__ void run_sink(const KArgs<F>& a, CtxT& ctx, BlockShared& sh, uint8_t* smem) {
    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    if (warp < kWarpsW) {
      for (int it = 0;; ++it) {
        const int b = it & 1;
        mbar_wait_sleep<direct_publish<F>(LO, HI, RTC) ? VP_BS_BACKOFF_NS : VP_MBAR_NS>(&sh.full[b], (uint32_t)((it >> 1) & 1));
        const int n = sh.bn[b];
        if (n < 0) break;
        ctx.ob = b;
        execute(a, ctx, sh, sh.bstage[b], in_buf(smem, b), n);
        __syncwarp();
        if (lane == 0) mbar_arrive(&sh.empty[b]);
      }
    } else if (warp == W_FETCH) {
      int last[2] = {0, 0};  // items of each buffer's last use, retired once it drains
      for (int it = 0;; ++it) {
        const int b = it & 1;
        if (it >= 2) {
          mbar_wait_sleep(&sh.empty[b], (uint32_t)(((it >> 1) - 1) & 1));
          if (lane == 0) sh.acc_neg -= last[b];
          last[b] = 0;
        }
        bool other_drained = it == 0;
        for (;;) {
          fetch(a, sh, smem, b, other_drained, lane);
          __syncwarp();
          if (sh.nx_n > 0 || sh.done) break;
          if (!other_drained) {
            // the block may be idle: the other buffer's batch must drain (and be retired)
            // before the termination test
            mbar_wait_sleep(&sh.empty[b ^ 1], (uint32_t)(((it - 1) >> 1) & 1));
            if (lane == 0) sh.acc_neg -= last[b ^ 1];
            last[b ^ 1] = 0;
            other_drained = true;
          }
        }
        const bool stop = sh.done && sh.nx_n == 0;
        last[b] = stop ? 0 : sh.nx_n;
        if (lane == 0) {
          sh.bn[b] = stop ? -1 : sh.nx_n;
          sh.bstage[b] = sh.nx_stage;
          sh.work[b] = 0;
          sh.rounds++;
          mbar_arrive(&sh.full[b]);
        }
        __syncwarp();
        if (stop) break;
      }
      // still-staged batches (abort path) are executed by the workers before they reach
      // the stop marker; they are retired here and flushed after the final block barrier
      if (lane == 0) sh.acc_neg -= last[0] + last[1];
    }
  }

  static __device__ void run(const KArgs<F>& a) {
    extern __shared__ __align__(128) uint8_t smem[];
    __shared__ BlockShared sh;
    const bool admitted = admit(a, sh);
    // cluster launch (work stealing): both CTAs learn whether the other was admitted, and
    // neither leaves before the other is done with its shared memory (final barrier)
    const bool clustered = kSteal && cluster_nctarank() == 2;
    if (clustered) {
      if (threadIdx.x == 0) sh.alive = admitted ? 1 : 0;
      cluster_sync_all();
      if (threadIdx.x == 0) sh.sib_alive = dsmem_ld_relaxed(dsmem_addr(&sh.alive, cluster_ctarank() ^ 1u));
      __syncthreads();
      if (!admitted) {
        cluster_sync_all();
        return;
      }
    }
    if (!admitted) return;
    CtxT ctx(a, smem, sh);
    if constexpr (sink_group()) {
      if (threadIdx.x == 0) {
        for (int b = 0; b < 2; ++b) {
          mbar_init(&sh.full[b], 1);
          mbar_init(&sh.empty[b], kWarpsW);
        }
      }
      if constexpr (scratch_of<F>(LO, HI, RTC) > 0) {
        for (int i = threadIdx.x; i < scratch_of<F>(LO, HI, RTC) / 4; i += blockDim.x) ((uint32_t*)ctx.scratch())[i] = 0u;
      }
      __syncthreads();
      run_sink(a, ctx, sh, smem);
      __syncthreads();
      flush_stats(a, sh);
      return;
    }
    if constexpr (scratch_of<F>(LO, HI, RTC) > 0) {  // family scratch starts zeroed
      for (int i = threadIdx.x; i < scratch_of<F>(LO, HI, RTC) / 4; i += blockDim.x) ((uint32_t*)ctx.scratch())[i] = 0u;
    }
    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    // prologue: stage the first batch into in[0]
    if (warp == W_FETCH) fetch(a, sh, smem, 0, true, lane);
    __syncthreads();
    int b = 0, prev_s = -1, prev_n = 0;
    for (;;) {
      const int done = sh.done, cur_s = sh.nx_stage, cur_n = sh.nx_n;
      // the previous round's users of the work counters finished at its end barrier; this
      // round's start after the next one
      if (threadIdx.x == 0) sh.work[0] = sh.work[1] = 0;
      __syncthreads();  // everyone has read the round's batch; the fetcher may overwrite it
      if (done) break;
      if (warp < kWarpsW) {
        if (cur_n > 0) {
          ctx.ob = b;
          execute(a, ctx, sh, cur_s, in_buf(smem, b), cur_n);
        }
      } else if (warp == W_FETCH) {
        fetch(a, sh, smem, b ^ 1, cur_n == 0 && prev_n == 0, lane);
      } else {
        if (prev_n > 0) publish(a, sh, smem, b ^ 1, prev_s, prev_n, lane);
      }
      __syncthreads();
      if (threadIdx.x == 0) sh.rounds++;
      prev_s = cur_s;
      prev_n = cur_n;
      b ^= 1;
    }
    flush_stats(a, sh);
    if (clustered) cluster_sync_all();
  }
};

template <class F, int LO, int HI, bool RTC>
__global__ void __launch_bounds__(Runner<F, LO, HI, RTC>::kBlockThreads, F::min_blocks(LO, HI, RTC))
    vp_kernel(const __grid_constant__ KArgs<F> a) {
  Runner<F, LO, HI, RTC>::run(a);
}

}  // namespace vp

// fam_qbench.cu — queue microbenchmark family (not a paper workload).
//
// Three independent self-recursive stages that differ only in their item size: 4 B (the
// toy's int, Fig. 9 L37), 16 B (the window / tile items of Table 2) and 272 B (the
// Reyes patch, "the largest data item structure in the queue", L61 §8.5).  A run seeds
// ONE of them.  Every item carries {id, remaining depth}; a non-leaf item emits `fanout`
// copies of itself one level down (fan-out 0: every seed is a leaf; 1: a chain of depth+1
// tasks; 2: a binary tree of 2^(depth+1)-1 tasks).  Children copy the whole payload, so
// every task moves stride bytes in and stride*fanout bytes out through the rings.  Leaves
// check the payload and add to per-stage counters (warp-aggregated).  The task count per
// seed is closed-form, which is what the tests pin.
#include "../../include/vp.h"
#include "vp_family.cuh"

namespace vp {

// One single-stage family per item size (round 2): a family's kernels reserve shared
// memory for every stage they cover, so three sizes in one family gave its megakernel the
// buffers of all three (1 block/SM) while a KBK wave kernel held one stage's (2 blocks/SM).
// K: 0 = 4 B, 1 = 16 B, 2 = 272 B; also the counter slot in vp_qbench_params.
// kSteal: the cluster-work-stealing variant (kinds VP_QB_ITEM{4,16}_CS) --
// a separate instantiation, so the plain kernels are not changed by the stealing code.
template <int K, bool kSteal = false>
struct QBenchF {
  static constexpr int S = 1;
  static constexpr int kinds[S] = {kSteal ? (K == 0 ? VP_QB_ITEM4_CS : VP_QB_ITEM16_CS)
                                          : (K == 0 ? VP_QB_ITEM4 : K == 1 ? VP_QB_ITEM16 : VP_QB_ITEM272)};
  using Params = vp_qbench_params;
  static constexpr int stride(int) { return K == 0 ? 4 : K == 1 ? 16 : 272; }
  static constexpr int threads_per_item(int) { return 1; }
  static constexpr int max_batch(int) { return K == 2 ? 64 : 1024; }
  static constexpr int default_batch(int) { return K == 2 ? 32 : 256; }
  static constexpr int fanout(int s, int t) { return s == t ? 2 : 0; }
  static constexpr bool rtc_ok(int, int) { return true; }
  static constexpr int kMaxBatch = 1024;
  static constexpr int scratch_bytes(int, int) { return 2 * kMaxBatch * 4; }
  static constexpr int default_cap_log2(int) { return 16; }  // callers size the seeded ring
  static constexpr int min_blocks(int, int, bool) { return 2; }
  // the two CTAs of a cluster may take items from each other's block-local queue (DSMEM;
  // with VP_FLAG_CLUSTER_STEAL)
  static constexpr bool kClusterSteal = kSteal;

  // word 0: id (low 24 bits) | remaining depth << 24; words 1..: payload(id, k)
  static __device__ __forceinline__ uint32_t payload(uint32_t id, int k) { return id * 2654435761u + (uint32_t)k * 40503u; }
  template <int s>
  static __device__ unsigned long long item_id(const uint8_t* it) {
    uint32_t w = *(const uint32_t*)it;
    return ((unsigned long long)(w >> 24) << 32) | (w & 0xffffffu);
  }

  // Block-cooperative task: (1) one thread per item decides leaf / inner and reserves its
  // children's out slots (one shared-memory atomic per warp); (2) one thread per (item,
  // 16-B chunk) copies the payload into the children or checks a leaf's payload; (3) the
  // per-item payload verdicts are counted (one global atomic per warp per counter).
  template <int s, class Ctx>
  static __device__ void exec(Ctx& ctx, const uint8_t* items, int n) {
    const Params& p = ctx.params();
    using V = typename Chunk<stride(s)>::T;
    constexpr int CW = Chunk<stride(s)>::per_item;   // chunks per item
    constexpr int EW = sizeof(V) / 4;                // words per chunk
    int* slot = (int*)ctx.scratch();                 // [kMaxBatch] first child slot, -1 = leaf
    int* badf = slot + kMaxBatch;                    // [kMaxBatch] leaf payload mismatch
    const int lane = threadIdx.x & 31;
    const uint32_t fan = p.fanout;
    for (int base = 0; base < n; base += kThreads) {
      const int k = base + threadIdx.x;
      const bool valid = k < n;
      uint32_t w0 = valid ? *(const uint32_t*)(items + (size_t)k * stride(s)) : 0u;
      const bool leaf = valid && (fan == 0 || (w0 >> 24) == 0);
      const int want = (valid && !leaf) ? (int)fan : 0;
      int incl = want;
#pragma unroll
      for (int o = 1; o < 32; o <<= 1) {
        int v = __shfl_up_sync(0xffffffffu, incl, o);
        if (lane >= o) incl += v;
      }
      const int total = __shfl_sync(0xffffffffu, incl, 31);
      int wbase = 0;
      if (lane == 0 && total > 0) wbase = ctx.template reserve<s>(total);
      wbase = __shfl_sync(0xffffffffu, wbase, 0);
      if (valid) {
        slot[k] = leaf ? -1 : (wbase < 0 ? -2 : wbase + incl - want);
        badf[k] = 0;
      }
      const unsigned lm = __ballot_sync(0xffffffffu, leaf);
      unsigned long long ids = leaf ? (unsigned long long)(w0 & 0xffffffu) : 0ull;
#pragma unroll
      for (int o = 16; o > 0; o >>= 1) ids += __shfl_xor_sync(0xffffffffu, ids, o);
      if (lane == 0 && lm) {
        atomicAdd(&p.leaves[K], (unsigned long long)__popc(lm));
        atomicAdd(&p.idsum[K], ids);
      }
    }
    worker_sync();
    for (int e = threadIdx.x; e < n * CW; e += kThreads) {
      const int k = e / CW, c = e - k * CW;
      V v = ((const V*)(items + (size_t)k * stride(s)))[c];
      uint32_t* w = (uint32_t*)&v;
      const int sl = slot[k];
      const uint32_t id = ((const uint32_t*)(items + (size_t)k * stride(s)))[0] & 0xffffffu;
      if (sl == -1) {
        bool bad = false;
#pragma unroll
        for (int j = 0; j < EW; ++j)
          if (c * EW + j > 0) bad |= w[j] != payload(id, c * EW + j);
        if (bad) badf[k] = 1;
      } else if (sl >= 0) {
        if (c == 0) w[0] = id | (((w[0] >> 24) - 1) << 24);
        for (uint32_t ch = 0; ch < fan; ++ch) ((V*)ctx.template out_ptr<s>(sl + (int)ch))[c] = v;
      }
    }
    worker_sync();
    for (int base = 0; base < n; base += kThreads) {
      const int k = base + threadIdx.x;
      const unsigned bm = __ballot_sync(0xffffffffu, k < n && badf[k] != 0);
      if (lane == 0 && bm) atomicAdd(&p.bad[K], (unsigned long long)__popc(bm));
    }
  }
  static cudaError_t init_run(const Params& p, cudaStream_t st) {
    cudaError_t e = cudaMemsetAsync(p.leaves, 0, 3 * sizeof(unsigned long long), st);
    if (e == cudaSuccess) e = cudaMemsetAsync(p.idsum, 0, 3 * sizeof(unsigned long long), st);
    if (e == cudaSuccess) e = cudaMemsetAsync(p.bad, 0, 3 * sizeof(unsigned long long), st);
    return e;
  }
  static cudaError_t finalize(const Params&, cudaStream_t) { return cudaSuccess; }
  static bool output(const Params& p, int idx, void** ptr, size_t* bytes) {
    if (idx == 0) { *ptr = p.leaves; *bytes = 24; return true; }
    if (idx == 1) { *ptr = p.idsum; *bytes = 24; return true; }
    if (idx == 2) { *ptr = p.bad; *bytes = 24; return true; }
    return false;
  }
  static const char* validate(const Params& p) {
    if (!p.leaves || !p.idsum || !p.bad) return "vp_qbench_params: leaves/idsum/bad must be device pointers";
    if (p.fanout > 2) return "vp_qbench_params: fanout must be 0, 1 or 2";
    if (p.depth > 255) return "vp_qbench_params: depth must be <= 255";
    if (p.fanout == 2 && p.depth > 30) return "vp_qbench_params: depth must be <= 30 with fan-out 2";
    return nullptr;
  }
};

const FamilyOps* family_qbench4() {
  static FamilyImpl<QBenchF<0>> f("qbench4");
  return &f;
}
const FamilyOps* family_qbench16() {
  static FamilyImpl<QBenchF<1>> f("qbench16");
  return &f;
}
const FamilyOps* family_qbench272() {
  static FamilyImpl<QBenchF<2>> f("qbench272");
  return &f;
}
const FamilyOps* family_qbench4_cs() {
  static FamilyImpl<QBenchF<0, true>> f("qbench4_cs");
  return &f;
}
const FamilyOps* family_qbench16_cs() {
  static FamilyImpl<QBenchF<1, true>> f("qbench16_cs");
  return &f;
}

}  // namespace vp

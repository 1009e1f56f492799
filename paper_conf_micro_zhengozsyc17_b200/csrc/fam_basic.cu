// fam_basic.cu — the Fig. 9 toy pipeline and the Collatz queue-stress
// pipeline (not in the paper), written as VersaPipe stage functions.
#include "../../include/vp.h"
#include "vp_family.cuh"

namespace vp {

// Warp-aggregated append to a global counter: one atomic per warp (Guideline 12).
__device__ __forceinline__ unsigned long long warp_append(unsigned long long* ctr, bool pred) {
  unsigned m = __ballot_sync(0xffffffffu, pred);
  if (!pred) return 0;
  int lane = threadIdx.x & 31;
  int leader = __ffs(m) - 1;
  unsigned long long base = 0;
  if (lane == leader) base = atomicAdd(ctr, (unsigned long long)__popc(m));
  base = __shfl_sync(m, base, leader);
  return base + __popc(m & ((1u << lane) - 1u));
}

// ---------------------------------------------------------------- toy (Fig. 9)
struct ToyF {
  static constexpr int S = 3;
  static constexpr int kinds[S] = {VP_TOY_S1, VP_TOY_S2, VP_TOY_S3};
  using Params = vp_toy_params;
  static constexpr int stride(int) { return 4; }               // typedef int DataItemType
  static constexpr int threads_per_item(int) { return 1; }     // int threadNum = 1
  static constexpr int max_batch(int) { return 1024; }
  static constexpr int default_batch(int) { return 256; }
  static constexpr int fanout(int s, int t) { return (s == 0 && (t == 0 || t == 1)) || (s == 1 && t == 2) ? 1 : 0; }
  static constexpr bool rtc_ok(int, int) { return true; }
  static constexpr int scratch_bytes(int, int) { return 0; }
  static constexpr int default_cap_log2(int) { return 20; }
  static constexpr int min_blocks(int, int, bool) { return 3; }
  template <int s>
  static __device__ unsigned long long item_id(const uint8_t* it) { return *(const uint32_t*)it; }

  template <int s, class Ctx>
  static __device__ void exec(Ctx& ctx, const uint8_t* items, int n) {
    const Params& p = ctx.params();
    for (int base = 0; base < n; base += kThreads) {
      int k = base + threadIdx.x;
      bool valid = k < n;
      int32_t v = valid ? ((const int32_t*)items)[k] : 0;
      if constexpr (s == 0) {  // Stage_1::execute: val *= 2; enqueue to stage 2 or back to 1
        if (valid) {
          v *= 2;
          if (v >= p.threshold) ctx.template emit<1>(&v);
          else ctx.template emit<0>(&v);
        }
      } else if constexpr (s == 1) {  // Stage_2 (reading R-T1): +1 -> stage 3
        if (valid) {
          v += 1;
          ctx.template emit<2>(&v);
        }
      } else {  // Stage_3: sink
        unsigned long long i = warp_append(p.n_out, valid);
        if (valid) p.out[i] = v;
      }
    }
  }
  static cudaError_t init_run(const Params& p, cudaStream_t st) {
    return cudaMemsetAsync(p.n_out, 0, sizeof(unsigned long long), st);
  }
  static cudaError_t finalize(const Params&, cudaStream_t) { return cudaSuccess; }
  static bool output(const Params& p, int idx, void** ptr, size_t* bytes) {
    if (idx == 0) { *ptr = p.out; *bytes = 0; return true; }
    if (idx == 1) { *ptr = p.n_out; *bytes = 8; return true; }
    return false;
  }
  static const char* validate(const Params& p) {
    if (!p.out || !p.n_out) return "vp_toy_params: out and n_out must be device pointers";
    if (p.threshold <= 0 || p.threshold > (1 << 30)) return "vp_toy_params: threshold must be in (0, 2^30]";
    return nullptr;
  }
};

// ---------------------------------------------------------------- Collatz stress
struct CollatzItem {
  uint32_t id, steps;
  unsigned long long v;
};

struct CollatzF {
  static constexpr int S = 2;
  static constexpr int kinds[S] = {VP_COLLATZ_STEP, VP_COLLATZ_SINK};
  using Params = vp_collatz_params;
  static constexpr int stride(int) { return 16; }
  static constexpr int threads_per_item(int) { return 1; }
  static constexpr int max_batch(int) { return 512; }
  static constexpr int default_batch(int) { return 256; }
  static constexpr int fanout(int s, int t) { return s == 0 ? 1 : 0; }
  static constexpr bool rtc_ok(int, int) { return true; }
  static constexpr int scratch_bytes(int, int) { return 0; }
  static constexpr int default_cap_log2(int) { return 20; }
  static constexpr int min_blocks(int, int, bool) { return 3; }
  template <int s>
  static __device__ unsigned long long item_id(const uint8_t* it) {
    const CollatzItem* c = (const CollatzItem*)it;
    return ((unsigned long long)c->id << 32) | c->steps;
  }
  template <int s, class Ctx>
  static __device__ void exec(Ctx& ctx, const uint8_t* items, int n) {
    const Params& p = ctx.params();
    for (int k = threadIdx.x; k < n; k += kThreads) {
      CollatzItem it = ((const CollatzItem*)items)[k];
      if constexpr (s == 0) {
        if (it.v == 1) {
          ctx.template emit<1>(&it);
        } else {
          if (it.steps >= p.max_steps) { ctx.abort(ABORT_GUARD); continue; }
          it.v = (it.v % 2 == 0) ? it.v / 2 : 3 * it.v + 1;
          it.steps++;
          ctx.template emit<0>(&it);
        }
      } else {
        if (it.id < p.n_ids) {
          p.steps_out[it.id] = it.steps;
          atomicAdd(&p.seen[it.id], 1u);
        }
      }
    }
  }
  static cudaError_t init_run(const Params& p, cudaStream_t st) {
    return cudaMemsetAsync(p.seen, 0, sizeof(uint32_t) * (size_t)p.n_ids, st);
  }
  static cudaError_t finalize(const Params&, cudaStream_t) { return cudaSuccess; }
  static bool output(const Params& p, int idx, void** ptr, size_t* bytes) {
    if (idx == 0) { *ptr = p.steps_out; *bytes = 4ull * p.n_ids; return true; }
    if (idx == 1) { *ptr = p.seen; *bytes = 4ull * p.n_ids; return true; }
    return false;
  }
  static const char* validate(const Params& p) {
    if (!p.steps_out || !p.seen || p.n_ids == 0) return "vp_collatz_params: steps_out/seen/n_ids required";
    return nullptr;
  }
};

const FamilyOps* family_toy() {
  static FamilyImpl<ToyF> f("toy");
  return &f;
}
const FamilyOps* family_collatz() {
  static FamilyImpl<CollatzF> f("collatz");
  return &f;
}

}  // namespace vp

// fam_ldpc.cu — the LDPC decoder of PAPER.md Fig. 17 (L59: "There are 4 stages in LDPC
// decoding pipeline" -- Initialize, C2V, V2C, ProbVar -- with an inner loop; L53: 100
// frames x 100 iterations; Table 1: Loop / Static; Table 2: 12-B items).  The
// paper takes its code from [18] and gives no arithmetic; readings R-L1..R-L6
// fix normalised min-sum on a regular H given as data (edge arrays in check-major order),
// float32 in a fixed operation order, so the results are bit-identical to the CPU oracle
// (compiled with -fmad=false).
//
// Items are {frame, iteration, chunk} (16-B slots, reading R-L6): Initialize is one item
// per frame; C2V, V2C and ProbVar items are chunks of <= 256 checks / variables (one per
// thread), so 100 frames give ~2000 items per iteration instead of 300.  Dependency
// latches join the chunks: the last C2V chunk of (f, it) emits the V2C and ProbVar chunks,
// the last of those emits the C2V chunks of (f, it + 1).  Message arrays live in global
// memory (L2-resident: 100 frames x 2 x 24 KB).
#include <math.h>

#include "../../include/vp.h"
#include "vp_family.cuh"

namespace vp {

struct LdpcItem {
  uint32_t frame, iter, chunk, pad;
};

// release this item's writes, count down; the last arriver acquires everybody's writes
__device__ __forceinline__ bool ldpc_latch_arrive(int* latch) {
  __threadfence();
  if (atomicSub(latch, 1) == 1) {
    __threadfence();
    return true;
  }
  return false;
}

struct LdpcF {
  static constexpr int S = 4;
  static constexpr int INIT = 0, C2V = 1, V2C = 2, PROBVAR = 3;
  static constexpr int kinds[S] = {VP_LDPC_INIT, VP_LDPC_C2V, VP_LDPC_V2C, VP_LDPC_PROBVAR};
  static constexpr int kMaxDc = 32, kMaxDv = 8, kMaxChunks = 16;
  using Params = vp_ldpc_params;
  static constexpr int stride(int) { return 16; }
  static constexpr int threads_per_item(int) { return kThreads; }
  static constexpr int max_batch(int) { return 4; }
  static constexpr int default_batch(int) { return 2; }
  // Init -> C2V chunks; last C2V chunk -> V2C + ProbVar chunks; last of those -> C2V
  // chunks of the next iteration (the inner loop of Fig. 17)
  static constexpr int fanout(int s, int t) {
    return (s == INIT && t == C2V) || (s == C2V && (t == V2C || t == PROBVAR)) || ((s == V2C || s == PROBVAR) && t == C2V)
               ? kMaxChunks
               : 0;
  }
  static constexpr bool rtc_ok(int, int) { return true; }
  static constexpr int scratch_bytes(int, int) { return 0; }
  static constexpr int default_cap_log2(int) { return 12; }
  static constexpr int min_blocks(int, int, bool) { return 4; }

  template <int s>
  static __device__ unsigned long long item_id(const uint8_t* it) {
    const LdpcItem* q = (const LdpcItem*)it;
    return ((unsigned long long)q->frame << 32) | ((unsigned long long)q->iter << 8) | q->chunk;
  }

  // check m: c2v[e] = sgn * (alpha * min over the other edges of |v2c|), reading R-L3.
  // DC > 0: compile-time degree (unrolled, registers); DC = 0: p.dc at run time (loops).
  static __device__ __forceinline__ void c2v_check(const Params& p, const float* x, int dc, int kk, float* out) {
    float mag = INFINITY;
    int neg = 0;
    for (int j = 0; j < dc; ++j) {
      if (j == kk) continue;
      const float a = fabsf(x[j]);
      if (a < mag) mag = a;
      neg ^= x[j] < 0.0f ? 1 : 0;
    }
    const float r = p.alpha * mag;
    *out = neg ? -r : r;
  }
  template <int DC>
  static __device__ __forceinline__ void c2v_frame(const Params& p, const float* v2c, float* c2v, int m0, int m1) {
    for (int m = m0 + (int)threadIdx.x; m < m1; m += kThreads) {
      if constexpr (DC > 0) {
        float x[DC];
#pragma unroll
        for (int j = 0; j < DC; ++j) x[j] = v2c[m * DC + j];
#pragma unroll
        for (int kk = 0; kk < DC; ++kk) c2v_check(p, x, DC, kk, &c2v[m * DC + kk]);
      } else {
        float x[kMaxDc];
        for (int j = 0; j < p.dc; ++j) x[j] = v2c[m * p.dc + j];
        for (int kk = 0; kk < p.dc; ++kk) c2v_check(p, x, p.dc, kk, &c2v[m * p.dc + kk]);
      }
    }
  }
  // variable v: v2c[e] = L + the other edges' c2v in edge order (reading R-L4)
  static __device__ __forceinline__ float v2c_sum(float l, const float* c, int dv, int kk) {
    float acc = l;
    for (int j = 0; j < dv; ++j)
      if (j != kk) acc = acc + c[j];
    return acc;
  }
  template <int DV>
  static __device__ __forceinline__ void v2c_frame(const Params& p, const float* L, const float* c2v, float* v2c, int n0,
                                                   int n1) {
    for (int v = n0 + (int)threadIdx.x; v < n1; v += kThreads) {
      if constexpr (DV > 0) {
        int eid[DV];
        float c[DV];
#pragma unroll
        for (int j = 0; j < DV; ++j) {
          eid[j] = __ldg(p.var_edges + v * DV + j);
          c[j] = c2v[eid[j]];
        }
        const float l = L[v];
#pragma unroll
        for (int kk = 0; kk < DV; ++kk) v2c[eid[kk]] = v2c_sum(l, c, DV, kk);
      } else {
        int eid[kMaxDv];
        float c[kMaxDv];
        for (int j = 0; j < p.dv; ++j) {
          eid[j] = __ldg(p.var_edges + v * p.dv + j);
          c[j] = c2v[eid[j]];
        }
        const float l = L[v];
        for (int kk = 0; kk < p.dv; ++kk) v2c[eid[kk]] = v2c_sum(l, c, p.dv, kk);
      }
    }
  }

  template <int s, class Ctx>
  static __device__ void exec(Ctx& ctx, const uint8_t* items, int n) {
    const Params& p = ctx.params();
    const int E = p.N * p.dv;
    for (int k = 0; k < n; ++k) {
      const LdpcItem it = ((const LdpcItem*)items)[k];
      if (it.frame >= (uint32_t)p.n_frames) continue;
      const float* L = p.llr + (size_t)it.frame * p.N;
      float* v2c = p.v2c + (size_t)it.frame * E;
      float* c2v = p.c2v + (size_t)it.frame * E;
      const int m0 = (int)((long long)it.chunk * p.M / p.nc_chk), m1 = (int)((long long)(it.chunk + 1) * p.M / p.nc_chk);
      const int n0 = (int)((long long)it.chunk * p.N / p.nc_var), n1 = (int)((long long)(it.chunk + 1) * p.N / p.nc_var);
      if constexpr (s == INIT) {
        for (int e = threadIdx.x; e < E; e += kThreads) v2c[e] = L[__ldg(p.check_vars + e)];
        if (threadIdx.x < p.nc_chk) {  // (visible through the publisher, after the round barrier)
          LdpcItem c{it.frame, 0u, threadIdx.x, 0u};
          ctx.template emit<C2V>(&c);
        }
      } else if constexpr (s == C2V) {
        if (p.dc == 6) c2v_frame<6>(p, v2c, c2v, m0, m1);  // the (3,6) code of the benchmark: registers only
        else c2v_frame<0>(p, v2c, c2v, m0, m1);
      } else if constexpr (s == V2C) {
        if (p.dv == 3) v2c_frame<3>(p, L, c2v, v2c, n0, n1);
        else v2c_frame<0>(p, L, c2v, v2c, n0, n1);
      } else {
        // posterior and hard decision against the all-zero codeword (reading R-L5)
        const bool last = (int)it.iter == p.n_iter - 1;
        int err = 0;
        for (int v = n0 + (int)threadIdx.x; v < n1; v += kThreads) {
          float acc = L[v];
          for (int j = 0; j < p.dv; ++j) acc = acc + c2v[__ldg(p.var_edges + v * p.dv + j)];
          err += acc < 0.0f ? 1 : 0;
          if (last) p.post[(size_t)it.frame * p.N + v] = acc;
        }
#pragma unroll
        for (int o = 16; o; o >>= 1) err += __shfl_xor_sync(0xffffffffu, err, o);
        if ((threadIdx.x & 31) == 0 && err) atomicAdd(p.errors + (size_t)it.frame * p.n_iter + it.iter, err);
      }
    }
    if constexpr (s != INIT) {
      // chunk joins (reading R-L6): after one barrier, thread k arrives for item k
      worker_sync();
      if ((int)threadIdx.x < n) {
        const LdpcItem it = ((const LdpcItem*)items)[threadIdx.x];
        if (it.frame < (uint32_t)p.n_frames) {
          if constexpr (s == C2V) {
            int* lat = p.latch + 2 * (size_t)it.frame;
            if (ldpc_latch_arrive(lat)) {
              atomicAdd(lat, p.nc_chk);  // re-arm for the next iteration before releasing
              for (int c = 0; c < p.nc_var; ++c) {
                LdpcItem x{it.frame, it.iter, (uint32_t)c, 0u};
                ctx.template emit<V2C>(&x);
                ctx.template emit<PROBVAR>(&x);
              }
            }
          } else {
            int* lat = p.latch + 2 * (size_t)it.frame + 1;
            if (ldpc_latch_arrive(lat)) {
              atomicAdd(lat, 2 * p.nc_var);
              if ((int)it.iter + 1 < p.n_iter)
                for (int c = 0; c < p.nc_chk; ++c) {
                  LdpcItem x{it.frame, it.iter + 1u, (uint32_t)c, 0u};
                  ctx.template emit<C2V>(&x);  // inner loop (Fig. 17)
                }
            }
          }
        }
      }
    }
  }

  static cudaError_t init_run(const Params& p, cudaStream_t st);
  static cudaError_t finalize(const Params&, cudaStream_t) { return cudaSuccess; }
  static bool output(const Params& p, int idx, void** ptr, size_t* bytes) {
    if (idx == 0) { *ptr = p.post; *bytes = 4ull * p.n_frames * p.N; return true; }
    if (idx == 1) { *ptr = p.errors; *bytes = 4ull * p.n_frames * p.n_iter; return true; }
    return false;
  }
  static const char* validate(const Params& p) {
    if (p.N <= 0 || p.M <= 0 || p.dv <= 0 || p.dc <= 1 || p.N * p.dv != p.M * p.dc) return "vp_ldpc_params: bad code shape";
    if (p.dc > kMaxDc || p.dv > kMaxDv) return "vp_ldpc_params: dc <= 32 and dv <= 8";
    if (p.n_frames <= 0 || p.n_iter <= 0) return "vp_ldpc_params: n_frames and n_iter must be positive";
    if (!p.check_vars || !p.var_edges || !p.llr || !p.v2c || !p.c2v || !p.post || !p.errors || !p.latch)
      return "vp_ldpc_params: all arrays are required device pointers";
    if (p.nc_chk < 1 || p.nc_var < 1 || p.nc_chk > kMaxChunks || p.nc_var > kMaxChunks || p.nc_chk > p.M || p.nc_var > p.N)
      return "vp_ldpc_params: 1 <= nc_chk, nc_var <= 16";
    return nullptr;
  }
};

__global__ void k_ldpc_init(vp_ldpc_params p) {
  for (int f = blockIdx.x * blockDim.x + threadIdx.x; f < p.n_frames; f += gridDim.x * blockDim.x) {
    p.latch[2 * f] = p.nc_chk;           // C2V chunks of the current iteration
    p.latch[2 * f + 1] = 2 * p.nc_var;   // V2C + ProbVar chunks
  }
}
cudaError_t LdpcF::init_run(const Params& p, cudaStream_t st) {
  cudaError_t e = cudaMemsetAsync(p.errors, 0, sizeof(int32_t) * (size_t)p.n_frames * p.n_iter, st);
  if (e != cudaSuccess) return e;
  k_ldpc_init<<<(p.n_frames + 255) / 256, 256, 0, st>>>(p);
  return cudaGetLastError();
}

const FamilyOps* family_ldpc() {
  static FamilyImpl<LdpcF> f("ldpc");
  return &f;
}

}  // namespace vp

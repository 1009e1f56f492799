// fam_cfd.cu — the CFD solver as VersaPipe stages (Fig. 15: Step Factor ->
// Flux -> Time Step, inner loop 3 / outer loop; L37: composite 1024-element items; Rodinia
// euler3d [8]).  Readings R-F1..R-F6.
//
// Items are tiles of T cells (1024 at G = 4096: a quarter row) at a global RK step k:
//   Copy(t, k=3o) -> StepFactor(t, k) -> [latch (t, k&1)] -> Flux(t, k) -> TimeStep(t, k)
//   -> arrivals on the Flux latches (t', k+1) of the tile and its neighbours, or, after the
//   third RK step, Copy(t, k+1) of the next outer iteration.
// The variables are ping-ponged by the parity of k, so a tile may start step k+1 as soon
// as its own and its neighbours' step k are done — no global barrier between RK steps.
// Arithmetic: bit-identical to the oracle (-fmad=false, same order).
#include <algorithm>

#include "../../include/vp.h"
#include "vp_family.cuh"

#ifndef VP_CFD_MINB
#define VP_CFD_MINB 3
#endif

namespace vp {

constexpr float kGamma = 1.4f, kSmooth = 0.2f;
constexpr int kRK = 3;

struct CfdItem {
  uint32_t tile, k, pad0, pad1;
};

struct CCell {
  float d, mx, my, mz, e;
};
struct CPrim {
  float vx, vy, vz, sq, c, p;
  float fmx[3], fmy[3], fmz[3], fe[3];
};

__device__ __forceinline__ void cfd_prim(const CCell& c, CPrim& q) {
  q.vx = c.mx / c.d;
  q.vy = c.my / c.d;
  q.vz = c.mz / c.d;
  float sq = q.vx * q.vx + q.vy * q.vy;
  q.sq = sq + q.vz * q.vz;
  q.p = (kGamma - 1.0f) * (c.e - 0.5f * c.d * q.sq);
  q.c = sqrtf(kGamma * q.p / c.d);
  q.fmx[0] = q.vx * c.mx + q.p;
  q.fmx[1] = q.vx * c.my;
  q.fmx[2] = q.vx * c.mz;
  q.fmy[0] = q.fmx[1];
  q.fmy[1] = q.vy * c.my + q.p;
  q.fmy[2] = q.vy * c.mz;
  q.fmz[0] = q.fmx[2];
  q.fmz[1] = q.fmy[2];
  q.fmz[2] = q.vz * c.mz + q.p;
  const float de_p = c.e + q.p;
  q.fe[0] = q.vx * de_p;
  q.fe[1] = q.vy * de_p;
  q.fe[2] = q.vz * de_p;
}

__device__ __forceinline__ CCell cfd_load(const float* v, size_t n, size_t i) {
  CCell c;
  c.d = __ldcg(v + i);
  c.mx = __ldcg(v + n + i);
  c.my = __ldcg(v + 2 * n + i);
  c.mz = __ldcg(v + 3 * n + i);
  c.e = __ldcg(v + 4 * n + i);
  return c;
}

__device__ __forceinline__ bool cfd_latch_arrive(int* latch) {
  __threadfence();
  if (atomicSub(latch, 1) == 1) {
    __threadfence();
    return true;
  }
  return false;
}

struct CfdF {
  static constexpr int S = 4;
  static constexpr int COPY = 0, STEP = 1, FLUX = 2, TIME = 3;
  static constexpr int kinds[S] = {VP_CFD_COPY, VP_CFD_STEP_FACTOR, VP_CFD_FLUX, VP_CFD_TIME_STEP};
  using Params = vp_cfd_params;
  static constexpr int stride(int) { return 16; }
  static constexpr int threads_per_item(int) { return 256; }
  static constexpr int max_batch(int s) { return s == FLUX ? 2 : 4; }
  static constexpr int default_batch(int s) { return max_batch(s); }
  static constexpr int fanout(int s, int t) {
    return (s == COPY && t == STEP) || (s == STEP && t == FLUX) || (s == FLUX && t == TIME) || (s == TIME && t == COPY) ? 1
           : (s == TIME && t == FLUX)                                                                           ? 5
                                                                                                                 : 0;
  }
  static constexpr bool rtc_ok(int, int) { return true; }  // back edges already exclude the loop
  static constexpr int scratch_bytes(int, int) { return 0; }
  static constexpr int default_cap_log2(int) { return 16; }
  static constexpr int min_blocks(int, int, bool) { return VP_CFD_MINB; }

  template <int s>
  static __device__ unsigned long long item_id(const uint8_t* it) {
    const CfdItem* c = (const CfdItem*)it;
    return ((unsigned long long)c->k << 32) | c->tile;
  }

  static __device__ __forceinline__ int tile_neighbours(const Params& p, uint32_t t, uint32_t nbt[4]) {
    const int tpr = p.G / p.T, r = (int)t / tpr, q = (int)t % tpr;
    int m = 0;
    if (q > 0) nbt[m++] = t - 1;
    if (q < tpr - 1) nbt[m++] = t + 1;
    if (r > 0) nbt[m++] = t - (uint32_t)tpr;
    if (r < p.G - 1) nbt[m++] = t + (uint32_t)tpr;
    return m;
  }

  template <class Ctx>
  static __device__ void arrive(Ctx& ctx, const Params& p, uint32_t t, uint32_t k) {
    int* lat = p.latch + (size_t)(k & 1u) * ((size_t)p.G * p.G / p.T) + t;
    if (cfd_latch_arrive(lat)) {
      uint32_t nbt[4];
      atomicAdd(lat, tile_neighbours(p, t, nbt) + 1);  // re-arm for k + 2 before releasing Flux(k)
      CfdItem f{t, k, 0, 0};
      ctx.template emit<FLUX>(&f);
    }
  }

  template <int s, class Ctx>
  static __device__ void exec(Ctx& ctx, const uint8_t* items, int n) {
    const Params& p = ctx.params();
    const size_t N = (size_t)p.G * p.G;
    for (int it = 0; it < n; ++it) {
      const CfdItem ci = ((const CfdItem*)items)[it];
      const size_t i0 = (size_t)ci.tile * p.T;
      const uint32_t k = ci.k;
      const float* cur = p.vars + (size_t)(k & 1u) * 5 * N;
      if constexpr (s == COPY) {
        for (int v = 0; v < 5; ++v)
          for (int i = threadIdx.x * 4; i < p.T; i += kThreads * 4)
            __stcg((float4*)(p.old + (size_t)v * N + i0 + i), __ldcg((const float4*)(cur + (size_t)v * N + i0 + i)));
        worker_sync();
        if (threadIdx.x == 0) ctx.template emit<STEP>(&ci);
      } else if constexpr (s == STEP) {
        for (int i = threadIdx.x; i < p.T; i += kThreads) {
          const size_t c = i0 + i;
          CCell cc = cfd_load(cur, N, c);
          CPrim q;
          cfd_prim(cc, q);
          p.sf[c] = 0.5f / (sqrtf(__ldg(p.area + c)) * (sqrtf(q.sq) + q.c));
        }
        worker_sync();
        if (threadIdx.x == 0) arrive(ctx, p, ci.tile, k);
      } else if constexpr (s == FLUX) {
        CCell ffc{p.ff[0], p.ff[1], p.ff[2], p.ff[3], p.ff[4]};
        CPrim qf;
        cfd_prim(ffc, qf);
        for (int i = threadIdx.x; i < p.T; i += kThreads) {
          const size_t c = i0 + i;
          const CCell ic = cfd_load(cur, N, c);
          CPrim qi;
          cfd_prim(ic, qi);
          const float speed_i = sqrtf(qi.sq);
          float fd = 0.0f, fe = 0.0f, fx = 0.0f, fy = 0.0f, fz = 0.0f;
#pragma unroll
          for (int j = 0; j < 4; ++j) {
            const int nb = __ldg(p.nb + (size_t)j * N + c);
            const float nx = __ldg(p.normals + ((size_t)j * 3 + 0) * N + c);
            const float ny = __ldg(p.normals + ((size_t)j * 3 + 1) * N + c);
            const float nz = __ldg(p.normals + ((size_t)j * 3 + 2) * N + c);
            float nlen = nx * nx + ny * ny;
            nlen = sqrtf(nlen + nz * nz);
            const float nn[3] = {nx, ny, nz};
            if (nb >= 0) {
              const CCell cn = cfd_load(cur, N, (size_t)nb);
              CPrim qn;
              cfd_prim(cn, qn);
              float factor = -nlen * kSmooth * 0.5f * (speed_i + sqrtf(qn.sq) + qi.c + qn.c);
              fd += factor * (ic.d - cn.d);
              fe += factor * (ic.e - cn.e);
              fx += factor * (ic.mx - cn.mx);
              fy += factor * (ic.my - cn.my);
              fz += factor * (ic.mz - cn.mz);
              const float mn[3] = {cn.mx, cn.my, cn.mz}, mi[3] = {ic.mx, ic.my, ic.mz};
#pragma unroll
              for (int a = 0; a < 3; ++a) {
                factor = 0.5f * nn[a];
                fd += factor * (mn[a] + mi[a]);
                fe += factor * (qn.fe[a] + qi.fe[a]);
                fx += factor * (qn.fmx[a] + qi.fmx[a]);
                fy += factor * (qn.fmy[a] + qi.fmy[a]);
                fz += factor * (qn.fmz[a] + qi.fmz[a]);
              }
            } else if (nb == -1) {
              fx += nx * qi.p;
              fy += ny * qi.p;
              fz += nz * qi.p;
            } else if (nb == -2) {
              const float mf[3] = {ffc.mx, ffc.my, ffc.mz}, mi[3] = {ic.mx, ic.my, ic.mz};
#pragma unroll
              for (int a = 0; a < 3; ++a) {
                const float factor = 0.5f * nn[a];
                fd += factor * (mf[a] + mi[a]);
                fe += factor * (qf.fe[a] + qi.fe[a]);
                fx += factor * (qf.fmx[a] + qi.fmx[a]);
                fy += factor * (qf.fmy[a] + qi.fmy[a]);
                fz += factor * (qf.fmz[a] + qi.fmz[a]);
              }
            }
          }
          __stcg(p.flux + c, fd);
          __stcg(p.flux + N + c, fx);
          __stcg(p.flux + 2 * N + c, fy);
          __stcg(p.flux + 3 * N + c, fz);
          __stcg(p.flux + 4 * N + c, fe);
        }
        worker_sync();
        if (threadIdx.x == 0) ctx.template emit<TIME>(&ci);
      } else {  // TimeStep
        const int rk = (int)(k % kRK);
        const uint32_t outer = k / kRK;
        float* nxt = p.vars + (size_t)((k + 1) & 1u) * 5 * N;
        const float denom = (float)(kRK + 1 - rk);
        for (int i = threadIdx.x * 4; i < p.T; i += kThreads * 4) {
          const size_t c = i0 + i;
          const float4 sf = __ldcg((const float4*)(p.sf + c));
          float4 f4;
          f4.x = sf.x / denom;
          f4.y = sf.y / denom;
          f4.z = sf.z / denom;
          f4.w = sf.w / denom;
          for (int v = 0; v < 5; ++v) {
            const float4 o = __ldcg((const float4*)(p.old + (size_t)v * N + c));
            const float4 fl = __ldcg((const float4*)(p.flux + (size_t)v * N + c));
            float4 r;
            r.x = o.x + f4.x * fl.x;
            r.y = o.y + f4.y * fl.y;
            r.z = o.z + f4.z * fl.z;
            r.w = o.w + f4.w * fl.w;
            __stcg((float4*)(nxt + (size_t)v * N + c), r);
          }
        }
        worker_sync();
        if (threadIdx.x == 0 && outer + (rk == kRK - 1 ? 1u : 0u) < (uint32_t)p.n_outer) {
          uint32_t nbt[4];
          const int m = tile_neighbours(p, ci.tile, nbt);
          for (int j = 0; j < m; ++j) arrive(ctx, p, nbt[j], k + 1);
          if (rk < kRK - 1) {
            arrive(ctx, p, ci.tile, k + 1);
          } else {
            CfdItem cp{ci.tile, k + 1, 0, 0};
            ctx.template emit<COPY>(&cp);
          }
        }
      }
      worker_sync();
    }
  }

  static cudaError_t init_run(const Params& p, cudaStream_t st);
  static cudaError_t finalize(const Params&, cudaStream_t) { return cudaSuccess; }
  static bool output(const Params& p, int idx, void** ptr, size_t* bytes) {
    const size_t N = (size_t)p.G * p.G;
    if (idx == 0) {
      *ptr = p.vars + (size_t)((3u * (unsigned)p.n_outer) & 1u) * 5 * N;
      *bytes = 5 * N * 4;
      return true;
    }
    return false;
  }
  static const char* validate(const Params& p) {
    if (p.G < 4 || p.T < 4 || p.T > p.G || p.G % p.T || p.T % 4) return "vp_cfd_params: T must divide G, T % 4 == 0";
    if (p.n_outer < 0) return "vp_cfd_params: n_outer >= 0";
    if (!p.vars0 || !p.vars || !p.old || !p.sf || !p.flux || !p.area || !p.nb || !p.normals || !p.latch)
      return "vp_cfd_params: all buffers are required";
    if (((uintptr_t)p.vars | (uintptr_t)p.old | (uintptr_t)p.sf | (uintptr_t)p.flux) & 15)
      return "vp_cfd_params: vars, old, sf, flux must be 16-B aligned";
    return nullptr;
  }
};

__global__ void k_cfd_init(vp_cfd_params p) {
  const size_t ntiles = (size_t)p.G * p.G / p.T;
  const int tpr = p.G / p.T;
  for (size_t t = blockIdx.x * (size_t)blockDim.x + threadIdx.x; t < ntiles; t += (size_t)gridDim.x * blockDim.x) {
    const int r = (int)(t / tpr), q = (int)(t % tpr);
    const int nbc = (q > 0) + (q < tpr - 1) + (r > 0) + (r < p.G - 1);
    p.latch[t] = 1;                  // k = 0: initial values are final; only StepFactor arrives
    p.latch[ntiles + t] = nbc + 1;   // k = 1
  }
}

cudaError_t CfdF::init_run(const Params& p, cudaStream_t st) {
  const size_t N = (size_t)p.G * p.G;
  cudaError_t e = cudaMemcpyAsync(p.vars, p.vars0, 5 * N * sizeof(float), cudaMemcpyDeviceToDevice, st);
  if (e != cudaSuccess) return e;
  k_cfd_init<<<148, 256, 0, st>>>(p);
  return cudaGetLastError();
}

const FamilyOps* family_cfd() {
  static FamilyImpl<CfdF> f("cfd");
  return &f;
}

}  // namespace vp

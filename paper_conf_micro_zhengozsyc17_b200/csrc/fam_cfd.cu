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

// a / b, exactly (IEEE round-to-nearest).  A zero dividend over a finite nonzero divisor
// is the signed zero, returned without the division: the IEEE division sequence takes its
// slow path for a zero dividend, and momentum components are exactly zero here (rho*w is
// 0 everywhere on this mesh; rho*v is 0 in the free stream).
__device__ __forceinline__ float div_rn_zero(float a, float b) {
  if (a == 0.0f && b != 0.0f && fabsf(b) <= 3.402823466e38f)
    return __uint_as_float((__float_as_uint(a) ^ __float_as_uint(b)) & 0x80000000u);
  return a / b;
}

__device__ __forceinline__ void cfd_prim(const CCell& c, CPrim& q) {
  q.vx = div_rn_zero(c.mx, c.d);
  q.vy = div_rn_zero(c.my, c.d);
  q.vz = div_rn_zero(c.mz, c.d);
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

__device__ __forceinline__ float f4_at(const float4& v, int i) { return i == 0 ? v.x : i == 1 ? v.y : i == 2 ? v.z : v.w; }

struct CfdF {
  static constexpr int S = 4;
  static constexpr int COPY = 0, STEP = 1, FLUX = 2, TIME = 3;
  static constexpr int kinds[S] = {VP_CFD_COPY, VP_CFD_STEP_FACTOR, VP_CFD_FLUX, VP_CFD_TIME_STEP};
  using Params = vp_cfd_params;
  static constexpr int stride(int) { return 16; }
  static constexpr int threads_per_item(int) { return 256; }
  static constexpr int max_batch(int s) { return s == FLUX ? 2 : 8; }
  static constexpr int default_batch(int s) { return max_batch(s); }
  static constexpr int fanout(int s, int t) {
    return (s == COPY && t == STEP) || (s == STEP && t == FLUX) || (s == FLUX && t == TIME) || (s == TIME && t == COPY) ? 1
           : (s == TIME && t == FLUX)                                                                           ? 5
                                                                                                                 : 0;
  }
  static constexpr bool rtc_ok(int, int) { return true; }  // back edges already exclude the loop
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

  // Flux shares one primitive-variable record per cell through shared memory, so a cell's
  // primitives are computed once per chunk instead of once per face that sees it
  // (Rodinia recomputes them per face; the values are identical, every op is the same).
  static constexpr int kShare = 20;        // d mx my mz e | speed c p | fmx[3] fmy[3] fmz[3] fe[3]
  static constexpr int kHalo = 8;          // left/right halo cell per chunk, <= 4 chunks per item
  static constexpr int kLd = kThreads + kHalo;
  // two chunk buffers (chunk parity) + the halo records: one barrier per chunk
  static constexpr int scratch_bytes(int lo, int hi) { return (lo <= FLUX && FLUX <= hi) ? kShare * (kLd + kThreads) * 4 : 0; }

  // Records are 20-float structures (five float4, 80 B apart: the 8 lanes of each
  // 128-bit shared-memory phase hit 8 distinct 4-bank groups, conflict-free).
  //   [d mx my mz] [e speed c p] [fmx0 fmx1 fmx2 fmy0] [fmy1 fmy2 fmz0 fmz1] [fmz2 fe0 fe1 fe2]
  static __device__ __forceinline__ void share_put(float4* sh, int col, const CCell& c, const CPrim& q, float speed) {
    float4* r = sh + 5 * col;
    r[0] = make_float4(c.d, c.mx, c.my, c.mz);
    r[1] = make_float4(c.e, speed, q.c, q.p);
    r[2] = make_float4(q.fmx[0], q.fmx[1], q.fmx[2], q.fmy[0]);
    r[3] = make_float4(q.fmy[1], q.fmy[2], q.fmz[0], q.fmz[1]);
    r[4] = make_float4(q.fmz[2], q.fe[0], q.fe[1], q.fe[2]);
  }
  struct NbRec {
    float d, mx, my, mz, e, speed, c, fmx[3], fmy[3], fmz[3], fe[3];
  };
  static __device__ __forceinline__ void share_get(const float4* sh, int col, NbRec& r) {
    const float4* q = sh + 5 * col;
    const float4 a = q[0], b = q[1], f2 = q[2], f3 = q[3], f4 = q[4];
    r.d = a.x; r.mx = a.y; r.my = a.z; r.mz = a.w;
    r.e = b.x; r.speed = b.y; r.c = b.z;
    r.fmx[0] = f2.x; r.fmx[1] = f2.y; r.fmx[2] = f2.z;
    r.fmy[0] = f2.w; r.fmy[1] = f3.x; r.fmy[2] = f3.y;
    r.fmz[0] = f3.z; r.fmz[1] = f3.w; r.fmz[2] = f4.x;
    r.fe[0] = f4.y; r.fe[1] = f4.z; r.fe[2] = f4.w;
  }
  // offsets are 32-bit: validate() bounds 16 * N < 2^31
  static __device__ __forceinline__ void gather(const float* cur, uint32_t N, uint32_t nb, NbRec& r) {
    const CCell cn{cur[nb], cur[N + nb], cur[2 * N + nb], cur[3 * N + nb], cur[4 * N + nb]};
    CPrim qn;
    cfd_prim(cn, qn);
    r.d = cn.d; r.mx = cn.mx; r.my = cn.my; r.mz = cn.mz; r.e = cn.e;
    r.speed = sqrtf(qn.sq);
    r.c = qn.c;
#pragma unroll
    for (int a = 0; a < 3; ++a) {
      r.fmx[a] = qn.fmx[a]; r.fmy[a] = qn.fmy[a]; r.fmz[a] = qn.fmz[a]; r.fe[a] = qn.fe[a];
    }
  }

  // Rodinia compute_flux over one tile item (orc_cfd_flux_cell, the same operation order).
  // Plain (L1-cacheable) loads of `cur` are coherent here: the item was acquired from its
  // ring after the producers' release (and the acquire invalidates L1), and the workers are
  // ordered after the fetcher by the round barrier.
  template <class Ctx>
  static __device__ void flux_item(Ctx& ctx, const Params& p, const CfdItem& ci) {
    const size_t N = (size_t)p.G * p.G;
    const float* cur = p.vars + (size_t)(ci.k & 1u) * 5 * N;
    const size_t i0 = (size_t)ci.tile * p.T;
    float4* sh = (float4*)ctx.scratch();
    const int t = threadIdx.x, nchunks = (p.T + kThreads - 1) / kThreads;
    const CCell ffc{p.ff[0], p.ff[1], p.ff[2], p.ff[3], p.ff[4]};
    // halo records: chunk h/2's left (h even) or right (h odd) neighbour cell, one per warp
    if ((t & 31) == 0 && (t >> 5) < 2 * nchunks) {
      const int h = t >> 5, ch = h >> 1;
      const long long lo = (long long)i0 + (long long)ch * kThreads;
      const long long hi = lo + min(kThreads, p.T - ch * kThreads);
      const long long cell = (h & 1) ? hi : lo - 1;
      if (cell >= 0 && cell < (long long)N) {
        NbRec r;
        gather(cur, (uint32_t)N, (uint32_t)cell, r);
        const CCell cc{r.d, r.mx, r.my, r.mz, r.e};
        CPrim q;
        q.c = r.c; q.p = 0.0f;
#pragma unroll
        for (int a = 0; a < 3; ++a) { q.fmx[a] = r.fmx[a]; q.fmy[a] = r.fmy[a]; q.fmz[a] = r.fmz[a]; q.fe[a] = r.fe[a]; }
        share_put(sh, kThreads + h, cc, q, r.speed);
      }
    }
    const uint32_t N32 = (uint32_t)N;
    for (int c0 = 0; c0 < p.T; c0 += kThreads) {
      const int nch = min(kThreads, p.T - c0), chunk = c0 / kThreads;
      const long long lo = (long long)i0 + c0, hi = lo + nch;
      const bool act = t < nch;
      const int buf = (chunk & 1) ? kLd : 0;  // this chunk's record columns
      const uint32_t c = (uint32_t)lo + (act ? t : 0);
      // this cell's faces: neighbour ids and normals are loaded before the barrier, so
      // their latency overlaps the primitive-variable computation
      int nbv[4];
      float nrm[4][3];
      if (act) {
        const CCell ic{cur[c], cur[N32 + c], cur[2 * N32 + c], cur[3 * N32 + c], cur[4 * N32 + c]};
#pragma unroll
        for (int j = 0; j < 4; ++j) {
          nbv[j] = __ldg(p.nb + (j * N32 + c));
#pragma unroll
          for (int a = 0; a < 3; ++a) nrm[j][a] = __ldg(p.normals + ((j * 3 + a) * N32 + c));
        }
        CPrim qi;
        cfd_prim(ic, qi);
        share_put(sh, buf + t, ic, qi, sqrtf(qi.sq));
      }
      worker_sync();
      if (act) {
        // this cell's record is read back from shared memory where it is used (registers
        // are the limit here: 3 resident blocks of 320 threads)
        const float4* me = sh + 5 * (buf + t);
#define ME(f) f4_at(me[(f) >> 2], (f) & 3)
        float fd = 0.0f, fe = 0.0f, fx = 0.0f, fy = 0.0f, fz = 0.0f;
#pragma unroll
        for (int j = 0; j < 4; ++j) {
          const int nb = nbv[j];
          const float nx = nrm[j][0], ny = nrm[j][1], nz = nrm[j][2];
          float nlen = nx * nx + ny * ny;
          nlen = sqrtf(nlen + nz * nz);
          const float nn[3] = {nx, ny, nz};
          if (nb >= 0) {
            int col = -1;
            if ((long long)nb >= lo && (long long)nb < hi) col = buf + (int)((long long)nb - lo);
            else if ((long long)nb == lo - 1) col = kThreads + 2 * chunk;
            else if ((long long)nb == hi) col = kThreads + 2 * chunk + 1;
            NbRec r;
            if (col >= 0) share_get(sh, col, r);
            else gather(cur, N32, (uint32_t)nb, r);
            float factor = -nlen * kSmooth * 0.5f * (ME(5) + r.speed + ME(6) + r.c);
            fd += factor * (ME(0) - r.d);
            fe += factor * (ME(4) - r.e);
            fx += factor * (ME(1) - r.mx);
            fy += factor * (ME(2) - r.my);
            fz += factor * (ME(3) - r.mz);
            const float mn[3] = {r.mx, r.my, r.mz};
#pragma unroll
            for (int a = 0; a < 3; ++a) {
              factor = 0.5f * nn[a];
              fd += factor * (mn[a] + ME(1 + a));
              fe += factor * (r.fe[a] + ME(17 + a));
              fx += factor * (r.fmx[a] + ME(8 + a));
              fy += factor * (r.fmy[a] + ME(11 + a));
              fz += factor * (r.fmz[a] + ME(14 + a));
            }
          } else if (nb == -1) {
            fx += nx * ME(7);
            fy += ny * ME(7);
            fz += nz * ME(7);
          } else if (nb == -2) {
            CPrim qf;
            cfd_prim(ffc, qf);
            const float mf[3] = {ffc.mx, ffc.my, ffc.mz};
#pragma unroll
            for (int a = 0; a < 3; ++a) {
              const float factor = 0.5f * nn[a];
              fd += factor * (mf[a] + ME(1 + a));
              fe += factor * (qf.fe[a] + ME(17 + a));
              fx += factor * (qf.fmx[a] + ME(8 + a));
              fy += factor * (qf.fmy[a] + ME(11 + a));
              fz += factor * (qf.fmz[a] + ME(14 + a));
            }
          }
        }
#undef ME
        __stcg(p.flux + c, fd);
        __stcg(p.flux + (N32 + c), fx);
        __stcg(p.flux + (2 * N32 + c), fy);
        __stcg(p.flux + (3 * N32 + c), fz);
        __stcg(p.flux + (4 * N32 + c), fe);
      }
      // no second barrier: chunk + 1 writes the other buffer, and chunk + 2's barrier
      // orders this chunk's reads before its buffer is rewritten
    }
    worker_sync();  // the next item rewrites the halo records and buffer 0
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
        // all five loads in flight before the stores (the arrays do not alias)
        for (int i = threadIdx.x * 4; i < p.T; i += kThreads * 4) {
          float4 v[5];
#pragma unroll
          for (int q = 0; q < 5; ++q) v[q] = *(const float4*)(cur + (size_t)q * N + i0 + i);
#pragma unroll
          for (int q = 0; q < 5; ++q) __stcg((float4*)(p.old + (size_t)q * N + i0 + i), v[q]);
        }
        // the emitted item becomes visible only through the publisher, after the round
        // barrier: no barrier is needed here
        if (threadIdx.x == 0) ctx.template emit<STEP>(&ci);
      } else if constexpr (s == STEP) {
        for (int i = threadIdx.x * 4; i < p.T; i += kThreads * 4) {
          const size_t c = i0 + i;
          float4 v[5];
#pragma unroll
          for (int q = 0; q < 5; ++q) v[q] = *(const float4*)(cur + (size_t)q * N + c);
          const float4 ar = __ldg((const float4*)(p.area + c));
          const float* vf = (const float*)v;
          const float* af = (const float*)&ar;
          float4 r;
          float* rf = (float*)&r;
#pragma unroll
          for (int u = 0; u < 4; ++u) {
            const CCell cc{vf[u], vf[4 + u], vf[8 + u], vf[12 + u], vf[16 + u]};
            CPrim q;
            cfd_prim(cc, q);
            rf[u] = 0.5f / (sqrtf(af[u]) * (sqrtf(q.sq) + q.c));
          }
          __stcg((float4*)(p.sf + c), r);
        }
      } else if constexpr (s == FLUX) {
        flux_item(ctx, p, ci);
        if (threadIdx.x == 0) ctx.template emit<TIME>(&ci);
      } else {  // TimeStep
        const int rk = (int)(k % kRK);
        const uint32_t outer = k / kRK;
        float* nxt = p.vars + (size_t)((k + 1) & 1u) * 5 * N;
        const float denom = (float)(kRK + 1 - rk);
        for (int i = threadIdx.x * 4; i < p.T; i += kThreads * 4) {
          const size_t c = i0 + i;
          // every load in flight before any store (old / flux / sf never alias nxt)
          const float4 sf = *(const float4*)(p.sf + c);
          float4 o[5], fl[5];
#pragma unroll
          for (int v = 0; v < 5; ++v) {
            o[v] = *(const float4*)(p.old + (size_t)v * N + c);
            fl[v] = *(const float4*)(p.flux + (size_t)v * N + c);
          }
          float4 f4;
          f4.x = sf.x / denom;
          f4.y = sf.y / denom;
          f4.z = sf.z / denom;
          f4.w = sf.w / denom;
#pragma unroll
          for (int v = 0; v < 5; ++v) {
            float4 r;
            r.x = o[v].x + f4.x * fl[v].x;
            r.y = o[v].y + f4.y * fl[v].y;
            r.z = o[v].z + f4.z * fl[v].z;
            r.w = o[v].w + f4.w * fl[v].w;
            __stcg((float4*)(nxt + (size_t)v * N + c), r);
          }
        }
      }
      // (Flux ends with a barrier of its own; Copy / StepFactor / TimeStep items write
      // disjoint tiles, so the next item's loads overlap this item's stores)
    }
    // Latch arrivals of the whole batch after ONE barrier (every thread's writes of every
    // item precede them), all in parallel: their fences and atomics overlap.
    if constexpr (s == STEP) {
      worker_sync();
      if ((int)threadIdx.x < n) {
        const CfdItem ci = ((const CfdItem*)items)[threadIdx.x];
        arrive(ctx, p, ci.tile, ci.k);
      }
    } else if constexpr (s == TIME) {
      worker_sync();
      // per item: thread j < m arrives on neighbour j, thread m on the tile itself (or
      // emits the next outer iteration's Copy)
      if ((int)threadIdx.x < 5 * n) {
        const CfdItem ci = ((const CfdItem*)items)[threadIdx.x / 5];
        const int j = threadIdx.x % 5;
        const uint32_t k = ci.k;
        const int rk = (int)(k % kRK);
        const uint32_t outer = k / kRK;
        if (outer + (rk == kRK - 1 ? 1u : 0u) < (uint32_t)p.n_outer) {
          uint32_t nbt[4];
          const int m = tile_neighbours(p, ci.tile, nbt);
          if (j < m) {
            arrive(ctx, p, nbt[j], k + 1);
          } else if (j == m) {
            if (rk < kRK - 1) {
              arrive(ctx, p, ci.tile, k + 1);
            } else {
              CfdItem cp{ci.tile, k + 1, 0, 0};
              ctx.template emit<COPY>(&cp);
            }
          }
        }
      }
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
    if ((long long)p.G * p.G * 16 >= (1ll << 31)) return "vp_cfd_params: G <= 8191 (32-bit cell offsets)";
    if (p.T > kThreads * (kHalo / 2)) return "vp_cfd_params: T <= 1024 (four 256-cell Flux chunks per item)";
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

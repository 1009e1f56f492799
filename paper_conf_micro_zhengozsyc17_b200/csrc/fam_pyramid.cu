// fam_pyramid.cu — image pyramid as VersaPipe stages (Fig. 12: Grayscale ->
// Histogram Equalization -> Resize (recursive); L51: HistEq's serial part is 96.1% of the
// KBK time; L55: KBK splits HistEq into 3 kernels).  Readings R-P1..R-P6.
//
// Stages: Gray(64x64 tile) -> [latch: all level-0 tiles of the image] -> CDF(image) ->
// Map(image, 8-tile row segment) -> [latch per level-1 tile] -> Resize(level, tile) ->
// [latch per next-level tile] -> Resize ...  The dependency latches
// replace the KBK global synchronisations: the last arriving task enqueues the
// dependent task, so the whole batch of images flows through one persistent run.
//
// HBM-bound stages (Gray, Map, Resize) move 16-B vectors; intermediate images are read
// with L1-bypassing loads (.cg) because other SMs produced them in the same run.
#include <algorithm>

#include "../../include/vp.h"
#include "vp_family.cuh"

#ifndef VP_PYR_PREFETCH  // Gray: load the next tile while converting this one, in every kernel
#define VP_PYR_PREFETCH 0  // measured: +16% time in the megakernel (register pressure), off;
#endif                     // a Gray-only kernel (KBK, or Gray as its own group) always prefetches
#ifndef VP_PYR_MINB
#define VP_PYR_MINB 3
#endif

namespace vp {

constexpr int kPT = 64;      // tile side
constexpr int kMapSeg = 8;   // level-0 tiles per Map item

struct PyrItem {
  uint32_t img, level, ty, tx;
};

__host__ __device__ __forceinline__ int pyr_levels(int S) {
  int L = 0;
  while ((S >> L) >= 1) ++L;
  return L;
}
__host__ __device__ __forceinline__ int pyr_tiles(int S, int l) {
  int s = S >> l;
  return s >= kPT ? s / kPT : 1;
}
__host__ __device__ __forceinline__ size_t pyr_level_off(int S, int l) {
  size_t off = 0;
  for (int k = 0; k < l; ++k) off += (size_t)(S >> k) * (size_t)(S >> k);
  return off;
}
// per-image pyramid stride: all levels, rounded up to 128 B so every image (and every
// level >= 64 px) starts 16-B aligned for the vector loads/stores
__host__ __device__ __forceinline__ size_t pyr_img_stride(int S) {
  size_t total = 0;
  for (int k = 0; (S >> k) >= 1; ++k) total += (size_t)(S >> k) * (size_t)(S >> k);
  return (total + 127) & ~(size_t)127;
}
// latch layout per image: [0] = CDF latch, then level l >= 1 tiles row-major
__host__ __device__ __forceinline__ size_t pyr_latch_off(int S, int l) {
  size_t n = 1;
  for (int k = 1; k < l; ++k) n += (size_t)pyr_tiles(S, k) * pyr_tiles(S, k);
  return n;
}
__host__ __device__ __forceinline__ size_t pyr_latches_per_img(int S) { return pyr_latch_off(S, pyr_levels(S)); }

// Dependency latch arrival (row a8): release our writes, count down; the last arriver
// acquires everybody's writes and returns true (it will enqueue the dependent task).
__device__ __forceinline__ bool latch_arrive(int* latch, int k) {
  __threadfence();
  int old = atomicSub(latch, k);
  if (old == k) {
    __threadfence();
    return true;
  }
  return false;
}

struct PyramidF {
  static constexpr int S = 4;
  static constexpr int GRAY = 0, CDF = 1, MAP = 2, RESIZE = 3;
  static constexpr int kMaxMap = 512;  // Map items per image for S <= 4096 (64 rows x 8 segments)
  static constexpr int kinds[S] = {VP_PYR_GRAY, VP_PYR_CDF, VP_PYR_MAP, VP_PYR_RESIZE};
  using Params = vp_pyramid_params;
  static constexpr int stride(int) { return 16; }
  static constexpr int threads_per_item(int) { return 256; }
  static constexpr int max_batch(int s) { return s == GRAY ? 16 : s == CDF ? 1 : s == MAP ? 4 : 8; }
  static constexpr int default_batch(int s) { return max_batch(s); }
  // Gray takes 16 tiles per claim only in its own kernel (the tile loads are pipelined
  // there, see gray_batch); kernels that also run later stages keep batches of 8
  static constexpr int kernel_max_batch(int lo, int hi, bool, int s) {
    return (s == GRAY && !(lo == GRAY && hi == GRAY)) ? 8 : max_batch(s);
  }
  static constexpr int fanout(int s, int t) {
    return (s == GRAY && t == CDF) ? 1 : (s == CDF && t == MAP) ? kMaxMap : (s == MAP && t == RESIZE) ? 4
                                                                        : (s == RESIZE && t == RESIZE) ? 1 : 0;
  }
  // CDF's fan-out must not be expanded block-locally from a batch of latch-fired items
  static constexpr bool rtc_ok(int lo, int hi) { return !(lo < CDF && hi >= CDF); }
  // sub-histograms / CDF / LUT staging, then the Map LUT-cache tag (image + 1, 0 = none)
  static constexpr int kLutTag = kWarpsW * 256 * 4;
  static constexpr int scratch_bytes(int, int) { return kLutTag + 16; }
  static __device__ __forceinline__ uint32_t* lut_tag(uint8_t* scratch) { return (uint32_t*)(scratch + kLutTag); }
  static constexpr int default_cap_log2(int s) { return s == MAP ? 16 : 15; }
  static constexpr int min_blocks(int, int, bool) { return VP_PYR_MINB; }

  template <int s>
  static __device__ unsigned long long item_id(const uint8_t* it) {
    const PyrItem* p = (const PyrItem*)it;
    return ((unsigned long long)p->img << 40) | ((unsigned long long)p->level << 32) | (p->ty << 16) | p->tx;
  }

  template <int s, class Ctx>
  static __device__ void exec(Ctx& ctx, const uint8_t* items, int n) {
    if constexpr (s == GRAY) {
      gray_batch(ctx, (const PyrItem*)items, n);
    } else if constexpr (s == MAP) {
      map_batch(ctx, (const PyrItem*)items, n);
    } else if constexpr (s == RESIZE) {
      resize_batch(ctx, (const PyrItem*)items, n);
    } else {
      for (int k = 0; k < n; ++k) {
        const PyrItem it = ((const PyrItem*)items)[k];
        if constexpr (s == CDF) cdf(ctx, it);
        else map(ctx, it);
        worker_sync();  // the block-wide stage functions reuse the scratch between items
      }
    }
  }

  // ------------------------------------------------------------ Gray (block per tile)
  // A batch of tiles accumulates into per-warp sub-histograms in shared memory (each
  // thread adds runs of equal values once), flushed to the image's global histogram when
  // the image changes and at the end of the batch; the CDF latch of every image is then
  // arrived on once with the batch's tile count for it.
  template <class Ctx>
  static __device__ void gray_batch(Ctx& ctx, const PyrItem* items, int n) {
    const Params& p = ctx.params();
    uint32_t* hs = (uint32_t*)ctx.scratch();  // [kWarpsW][256]
    const int t = threadIdx.x, w = t >> 5;
    if (t == 0) *lut_tag(ctx.scratch()) = 0u;  // the sub-histograms overwrite Map's cached LUT
    for (int i = t; i < kWarpsW * 256; i += kThreads) hs[i] = 0;
    worker_sync();
    const size_t npx = (size_t)p.S * p.S;
    const int y = t >> 2, x0 = (t & 3) * 16;  // thread t: 16 consecutive pixels of tile row t/4
    // the next tile's 48 B per thread are loaded while this tile is converted (two tiles
    // of loads in flight per block instead of one)
    auto load = [&](int k, uint4* v) {
      const PyrItem it = items[k];
      if (it.img < (uint32_t)p.n_img) {
        const size_t row = (size_t)(it.ty * kPT + y) * p.S + (size_t)it.tx * kPT + x0;
        const uint4* src = (const uint4*)(p.rgb + ((size_t)it.img * npx + row) * 3);
#pragma unroll
        for (int q = 0; q < 3; ++q) v[q] = __ldg(src + q);
      }
    };
    uint4 vn[3];
    constexpr bool kPrefetch = VP_PYR_PREFETCH || (Ctx::kLo == GRAY && Ctx::kHi == GRAY);
    if (kPrefetch && n > 0) load(0, vn);
    int k0 = 0;
    for (int k = 0; k < n; ++k) {
      const PyrItem it = items[k];
      uint4 v[3];
      if (kPrefetch) {
#pragma unroll
        for (int q = 0; q < 3; ++q) v[q] = vn[q];
        if (k + 1 < n) load(k + 1, vn);
      } else {
        load(k, v);
      }
      if (it.img < (uint32_t)p.n_img) {
        const size_t row = (size_t)(it.ty * kPT + y) * p.S + (size_t)it.tx * kPT + x0;
        const uint8_t* b = (const uint8_t*)v;
        __align__(16) uint8_t g[16];
#pragma unroll
        for (int i = 0; i < 16; ++i) g[i] = (uint8_t)((77u * b[3 * i] + 150u * b[3 * i + 1] + 29u * b[3 * i + 2] + 128u) >> 8);
        *(uint4*)(p.gray + (size_t)it.img * npx + row) = *(const uint4*)g;
        uint32_t cur = g[0], cnt = 1;
#pragma unroll
        for (int i = 1; i < 16; ++i) {
          if (g[i] == cur) {
            ++cnt;
          } else {
            atomicAdd(&hs[w * 256 + cur], cnt);
            cur = g[i];
            cnt = 1;
          }
        }
        atomicAdd(&hs[w * 256 + cur], cnt);
      }
      const bool last = k + 1 == n || items[k + 1].img != it.img;
      if (last) {  // flush the image's counts (block-uniform branch)
        worker_sync();
        if (it.img < (uint32_t)p.n_img) {
          uint32_t sum = 0;
#pragma unroll
          for (int q = 0; q < kWarpsW; ++q) {
            sum += hs[q * 256 + t];
            hs[q * 256 + t] = 0;
          }
          if (sum) atomicAdd(&p.hist[(size_t)it.img * 256 + t], sum);
        }
        worker_sync();
        if (t == 0 && it.img < (uint32_t)p.n_img &&
            latch_arrive(p.latch + (size_t)it.img * pyr_latches_per_img(p.S), k + 1 - k0)) {
          PyrItem c{it.img, 0, 0, 0};
          ctx.template emit<CDF>(&c);
        }
        k0 = k + 1;
      }
    }
  }

  // ------------------------------------------------------------ CDF (block per image)
  template <class Ctx>
  static __device__ void cdf(Ctx& ctx, const PyrItem& it) {
    const Params& p = ctx.params();
    if (it.img >= (uint32_t)p.n_img) return;
    uint32_t* cs = (uint32_t*)ctx.scratch();
    uint8_t* lut = ctx.scratch() + 256 * 4;
    const int t = threadIdx.x;
    if (t == 0) *lut_tag(ctx.scratch()) = 0u;  // lut below is this image's, but staged before it is final
    const uint32_t h = __ldcg(&p.hist[(size_t)it.img * 256 + t]);
    cs[t] = h;
    worker_sync();
    // inclusive scan (Hillis-Steele over 256 entries)
    for (int o = 1; o < 256; o <<= 1) {
      uint32_t v = t >= o ? cs[t - o] : 0u;
      worker_sync();
      cs[t] += v;
      worker_sync();
    }
    // first non-empty bin (worker-only barriers: the scheduler warps are elsewhere)
    __shared__ int first_s;
    if (t == 0) first_s = 256;
    worker_sync();
    if (h != 0u) atomicMin(&first_s, t);
    worker_sync();
    const int f = first_s;
    const unsigned long long N = (unsigned long long)p.S * p.S;
    const unsigned long long cmin = f < 256 ? cs[f] : 0ull;
    uint8_t v;
    if (N == cmin) v = (uint8_t)t;
    else if (t < f) v = 0;
    else v = (uint8_t)((((unsigned long long)cs[t] - cmin) * 255ull + (N - cmin) / 2ull) / (N - cmin));
    lut[t] = v;
    p.lut[(size_t)it.img * 256 + t] = v;
    worker_sync();
    // emit the Map items: nt rows x ceil(nt / 8) segments
    const int nt = pyr_tiles(p.S, 0), nseg = (nt + kMapSeg - 1) / kMapSeg, nm = nt * nseg;
    for (int m = t; m < nm; m += kThreads) {
      PyrItem q{it.img, 0, (uint32_t)(m / nseg), (uint32_t)((m % nseg) * kMapSeg)};
      ctx.template emit<MAP>(&q);
    }
  }

  // ------------------------------------------------------------ Map (level 0 = LUT[gray])
  // A batch of row segments: the LUT is staged in shared memory once per image (tagged,
  // so consecutive items and rounds of the same image reuse it), every segment's loads are
  // in flight before its lookups and stores, and the level-1 latch arrivals of the whole
  // batch happen together after one barrier (their fences and atomics overlap).
  template <class Ctx>
  static __device__ void map_batch(Ctx& ctx, const PyrItem* items, int n) {
    const Params& p = ctx.params();
    uint8_t* lut = ctx.scratch() + 256 * 4;
    uint32_t* tag = lut_tag(ctx.scratch());
    const int t = threadIdx.x;
    const int nt = pyr_tiles(p.S, 0);
    const size_t npx = (size_t)p.S * p.S, total = pyr_img_stride(p.S);
    for (int k = 0; k < n; ++k) {
      const PyrItem it = items[k];
      if (it.img >= (uint32_t)p.n_img) continue;  // block-uniform
      if (*tag != it.img + 1u) {  // block-uniform: everyone read the same tag
        worker_sync();            // nobody still reads the previous LUT
        lut[t] = __ldcg(p.lut + (size_t)it.img * 256 + t);
        worker_sync();
        if (t == 0) *tag = it.img + 1u;
      }
      const int tx1 = min((int)it.tx + kMapSeg, nt);
      const int wpx = (tx1 - (int)it.tx) * kPT;              // segment width in pixels
      const uint8_t* g = p.gray + (size_t)it.img * npx;
      uint8_t* dst = p.pyr + (size_t)it.img * total;
      const int vec_per_row = wpx / 16, nvec = kPT * vec_per_row;
      // up to 8 vectors per thread, all loads in flight before the lookups and stores
      constexpr int kV = kMapSeg * kPT * kPT / 16 / kThreads;
      uint4 v[kV];
#pragma unroll
      for (int u = 0; u < kV; ++u) {
        const int i = t + u * kThreads;
        if (i < nvec) {
          const int y = i / vec_per_row, xv = i - y * vec_per_row;
          v[u] = *(const uint4*)(g + (size_t)(it.ty * kPT + y) * p.S + (size_t)it.tx * kPT + xv * 16);
        }
      }
#pragma unroll
      for (int u = 0; u < kV; ++u) {
        const int i = t + u * kThreads;
        if (i < nvec) {
          const int y = i / vec_per_row, xv = i - y * vec_per_row;
          uint8_t* b = (uint8_t*)&v[u];
#pragma unroll
          for (int q = 0; q < 16; ++q) b[q] = lut[b[q]];
          *(uint4*)(dst + (size_t)(it.ty * kPT + y) * p.S + (size_t)it.tx * kPT + xv * 16) = v[u];
        }
      }
      worker_sync();  // the tag may be read again only after every thread read it for this item
    }
    // latch arrivals on level 1: each level-1 tile gets one count per source tile
    constexpr int kA = kMapSeg / 2 + 1;  // level-1 tiles a segment can touch
    if (pyr_levels(p.S) > 1 && t < n * kA) {
      const PyrItem it = items[t / kA];
      const int j = t % kA;
      if (it.img < (uint32_t)p.n_img) {
        const int tx1 = min((int)it.tx + kMapSeg, nt);
        const int a = (int)it.tx / 2 + j;                       // level-1 tile column
        const int c0 = max((int)it.tx, 2 * a), c1 = min(tx1, 2 * a + 2);
        const int k = c1 - c0;
        const int nt1 = pyr_tiles(p.S, 1);
        if (k > 0) {  // k > 0 implies a < nt1
          const int by = (int)it.ty / 2, bx = a;
          int* lat = p.latch + (size_t)it.img * pyr_latches_per_img(p.S) + pyr_latch_off(p.S, 1) + (size_t)by * nt1 + bx;
          if (latch_arrive(lat, k)) {
            PyrItem r{it.img, 1, (uint32_t)by, (uint32_t)bx};
            ctx.template emit<RESIZE>(&r);
          }
        }
      }
    }
  }

  // ------------------------------------------------------------ Resize (2x2 box)
  // The batch's tiles are independent (disjoint outputs): all are computed, then one
  // barrier, then thread k arrives on item k's next-level latch (the fences overlap).
  template <class Ctx>
  static __device__ void resize_batch(Ctx& ctx, const PyrItem* items, int n) {
    for (int k = 0; k < n; ++k) resize_tile(ctx, items[k]);
    worker_sync();
    const Params& p = ctx.params();
    const int t = threadIdx.x;
    if (t < n) {
      const PyrItem it = items[t];
      const int l = (int)it.level, L = pyr_levels(p.S);
      if (it.img < (uint32_t)p.n_img && l >= 1 && l + 1 < L) {
        const int nt1 = pyr_tiles(p.S, l + 1);
        const int by = (int)it.ty / 2, bx = (int)it.tx / 2;
        int* lat = p.latch + (size_t)it.img * pyr_latches_per_img(p.S) + pyr_latch_off(p.S, l + 1) + (size_t)by * nt1 + bx;
        if (latch_arrive(lat, 1)) {
          PyrItem r{it.img, (uint32_t)(l + 1), (uint32_t)by, (uint32_t)bx};
          ctx.template emit<RESIZE>(&r);
        }
      }
    }
  }

  template <class Ctx>
  static __device__ void resize_tile(Ctx& ctx, const PyrItem& it) {
    const Params& p = ctx.params();
    if (it.img >= (uint32_t)p.n_img) return;
    const int l = (int)it.level, L = pyr_levels(p.S);
    if (l < 1 || l >= L) return;
    const int s = p.S >> l, sp = p.S >> (l - 1), w = min(s, kPT);
    const size_t total = pyr_img_stride(p.S);
    uint8_t* base = p.pyr + (size_t)it.img * total;
    const uint8_t* src = base + pyr_level_off(p.S, l - 1);
    uint8_t* dst = base + pyr_level_off(p.S, l);
    const int t = threadIdx.x;
    if (w == kPT) {
      // thread t: 16 output pixels of row t/4 from 2 input rows of 32 bytes
      const int y = t >> 2, x0 = (t & 3) * 16;
      const int gy = (int)it.ty * kPT + y, gx = (int)it.tx * kPT + x0;
      const uint4* r0 = (const uint4*)(src + (size_t)(2 * gy) * sp + 2 * gx);
      const uint4* r1 = (const uint4*)(src + (size_t)(2 * gy + 1) * sp + 2 * gx);
      const uint4 a0 = r0[0], a1 = r0[1], b0 = r1[0], b1 = r1[1];
      __align__(16) uint8_t ra[32];
      __align__(16) uint8_t rb[32];
      __align__(16) uint8_t o[16];
      *(uint4*)ra = a0;
      *(uint4*)(ra + 16) = a1;
      *(uint4*)rb = b0;
      *(uint4*)(rb + 16) = b1;
#pragma unroll
      for (int i = 0; i < 16; ++i)
        o[i] = (uint8_t)(((unsigned)ra[2 * i] + ra[2 * i + 1] + rb[2 * i] + rb[2 * i + 1] + 2u) >> 2);
      *(uint4*)(dst + (size_t)gy * s + gx) = *(const uint4*)o;
    } else {
      for (int i = t; i < w * w; i += kThreads) {
        const int y = i / w, x = i - y * w;
        unsigned a = src[(size_t)(2 * y) * sp + 2 * x], b = src[(size_t)(2 * y) * sp + 2 * x + 1];
        unsigned c = src[(size_t)(2 * y + 1) * sp + 2 * x], d = src[(size_t)(2 * y + 1) * sp + 2 * x + 1];
        dst[(size_t)y * s + x] = (uint8_t)((a + b + c + d + 2u) >> 2);
      }
    }
  }

  static cudaError_t init_run(const Params& p, cudaStream_t st);
  static cudaError_t finalize(const Params&, cudaStream_t) { return cudaSuccess; }
  static bool output(const Params& p, int idx, void** ptr, size_t* bytes) {
    size_t total = pyr_img_stride(p.S);
    if (idx == 0) { *ptr = p.pyr; *bytes = total * (size_t)p.n_img; return true; }
    if (idx == 1) { *ptr = p.lut; *bytes = 256 * (size_t)p.n_img; return true; }
    return false;
  }
  static const char* validate(const Params& p) {
    if (p.S < kPT || p.S > 4096 || (p.S & (p.S - 1))) return "vp_pyramid_params: S must be a power of two in [64, 4096]";
    if (p.n_img <= 0 || p.n_img > (1 << 20)) return "vp_pyramid_params: bad n_img";
    if (!p.rgb || !p.gray || !p.pyr || !p.hist || !p.lut || !p.latch) return "vp_pyramid_params: all buffers are required";
    if (((uintptr_t)p.rgb & 15) || ((uintptr_t)p.gray & 15) || ((uintptr_t)p.pyr & 15))
      return "vp_pyramid_params: rgb, gray, pyr must be 16-B aligned";
    return nullptr;
  }
};

// Per run: zero the histograms, arm every latch with its number of source tiles.
__global__ void k_pyr_init(vp_pyramid_params p) {
  const size_t per = pyr_latches_per_img(p.S);
  const int L = pyr_levels(p.S);
  for (size_t i = blockIdx.x * (size_t)blockDim.x + threadIdx.x; i < per * (size_t)p.n_img;
       i += (size_t)gridDim.x * blockDim.x) {
    const size_t k = i % per;
    int v;
    if (k == 0) {
      v = pyr_tiles(p.S, 0) * pyr_tiles(p.S, 0);
    } else {
      int l = 1;
      while (l + 1 < L && k >= pyr_latch_off(p.S, l + 1)) ++l;
      const int src = pyr_tiles(p.S, l - 1) >= 2 ? 2 : 1;
      v = src * src;
    }
    p.latch[i] = v;
  }
  for (size_t i = blockIdx.x * (size_t)blockDim.x + threadIdx.x; i < 256 * (size_t)p.n_img;
       i += (size_t)gridDim.x * blockDim.x)
    p.hist[i] = 0;
}

cudaError_t PyramidF::init_run(const Params& p, cudaStream_t st) {
  k_pyr_init<<<148, 256, 0, st>>>(p);
  return cudaGetLastError();
}

const FamilyOps* family_pyramid() {
  static FamilyImpl<PyramidF> f("pyramid");
  return &f;
}

}  // namespace vp

// fam_facedet.cu — LBP face detection as VersaPipe stages (Fig. 14:
// Grayscale -> Histogram Equalization -> Resize (recursive) -> Feature Extraction ->
// Scanning; "the search window is the data item"; windows without faces end early).
// Readings R-D1..R-D8.
//
// Stages: Gray(band) -> [latch: frame] -> CDF(frame) -> Map(band) -> [latches] ->
// Resize(level, band) (recursive) ... LBP(level, band) -> [latch per window-row group]
// -> Scan(level, window row).  Bands are 32 rows; a Scan item is a row of windows
// (composite item, L37) evaluated one window per thread with early exit.
#include <algorithm>

#include "../../include/vp.h"
#include "vp_family.cuh"

#ifndef VP_FD_MINB
#define VP_FD_MINB 3
#endif

namespace vp {

constexpr int kBand = 32, kWin = 24, kMaxLev = 8;

struct FdItem {
  uint32_t frame, level, a, pad;  // a = band (Gray/Map/Resize/LBP) or window row (Scan)
};

struct FdGeo {
  int L;
  int W[kMaxLev], H[kMaxLev], nb[kMaxLev];
  size_t off[kMaxLev + 1];                                  // level offsets in a frame's pyramid
  size_t lat_rs[kMaxLev], lat_lbp[kMaxLev], lat_scan[kMaxLev], lat_per;  // latch layout
  __host__ __device__ FdGeo(int W0, int H0) {
    L = 0;
    int w = W0, h = H0;
    size_t o = 0;
    while (L < kMaxLev && w >= kWin && h >= kWin) {
      W[L] = w;
      H[L] = h;
      nb[L] = (h + kBand - 1) / kBand;
      off[L] = o;
      o += (size_t)w * h;
      ++L;
      w = (4 * w) / 5;
      h = (4 * h) / 5;
    }
    off[L] = o;
    size_t n = 1;
    for (int l = 0; l < L; ++l) lat_rs[l] = n, n += nb[l];
    for (int l = 0; l < L; ++l) lat_lbp[l] = n, n += nb[l];
    for (int l = 0; l < L; ++l) lat_scan[l] = n, n += nb[l];
    lat_per = n;
  }
  __host__ __device__ void resize_src(int l, int b, int& b0, int& b1) const {
    int y0 = b * kBand, y1 = min(y0 + kBand - 1, H[l] - 1);
    b0 = ((5 * y0) >> 2) / kBand;
    b1 = ((5 * y1) >> 2) / kBand;
  }
};

__device__ __forceinline__ uint8_t fd_gray(const uint8_t* rgb) {
  return (uint8_t)((77u * rgb[0] + 150u * rgb[1] + 29u * rgb[2] + 128u) >> 8);
}

__device__ __forceinline__ bool fd_latch(int* latch) {
  __threadfence();
  if (atomicSub(latch, 1) == 1) {
    __threadfence();
    return true;
  }
  return false;
}

struct FaceDetF {
  static constexpr int S = 6;
  static constexpr int GRAY = 0, CDF = 1, MAP = 2, RESIZE = 3, LBP = 4, SCAN = 5;
  static constexpr int kMaxBands0 = 64;  // H <= 2048
  static constexpr int kinds[S] = {VP_FD_GRAY, VP_FD_CDF, VP_FD_MAP, VP_FD_RESIZE, VP_FD_LBP, VP_FD_SCAN};
  using Params = vp_facedet_params;
  static constexpr int stride(int) { return 16; }
  static constexpr int threads_per_item(int) { return 256; }
  static constexpr int max_batch(int s) { return s == CDF ? 1 : s == SCAN ? 8 : 2; }
  static constexpr int default_batch(int s) { return max_batch(s); }
  static constexpr int fanout(int s, int t) {
    return (s == GRAY && t == CDF)       ? 1
           : (s == CDF && t == MAP)      ? kMaxBands0
           : (s == MAP && t == RESIZE)   ? 2
           : (s == MAP && t == LBP)      ? 3
           : (s == RESIZE && t == RESIZE) ? 2
           : (s == RESIZE && t == LBP)   ? 3
           : (s == LBP && t == SCAN)     ? 2 * kBand
                                         : 0;
  }
  static constexpr bool rtc_ok(int lo, int hi) { return !(lo < CDF && hi >= CDF); }
  static constexpr int scratch_bytes(int, int hi) { return hi >= SCAN ? kScanScratch : 6144; }
  static constexpr int default_cap_log2(int s) { return s == SCAN ? 15 : 13; }
  static constexpr int min_blocks(int, int, bool) { return VP_FD_MINB; }

  template <int s>
  static __device__ unsigned long long item_id(const uint8_t* it) {
    const FdItem* p = (const FdItem*)it;
    return ((unsigned long long)p->frame << 40) | ((unsigned long long)p->level << 32) | p->a;
  }

  static __device__ __forceinline__ int* latches(const Params& p, const FdGeo& g, uint32_t f) {
    return p.latch + (size_t)f * g.lat_per;
  }

  // image band (l, b) complete: LBP latches (l, b-1..b+1), Resize latches (l+1, b')
  template <class Ctx>
  static __device__ void image_band_done(Ctx& ctx, const Params& p, const FdGeo& g, uint32_t f, int l, int b) {
    int* lat = latches(p, g, f);
    for (int d = -1; d <= 1; ++d) {
      const int bb = b + d;
      if (bb < 0 || bb >= g.nb[l]) continue;
      if (fd_latch(lat + g.lat_lbp[l] + bb)) {
        FdItem it{f, (uint32_t)l, (uint32_t)bb, 0};
        ctx.template emit<LBP>(&it);
      }
    }
    if (l + 1 < g.L) {
      // level l+1 bands whose source rows include band b (at most two)
      const int lo = max(0, (kBand * b - 38 + 39) / 40 - 1), hi = min(g.nb[l + 1] - 1, (kBand * b + kBand - 1) / 40 + 1);
      for (int bb = lo; bb <= hi; ++bb) {
        int s0, s1;
        g.resize_src(l + 1, bb, s0, s1);
        if (b < s0 || b > s1) continue;
        if (fd_latch(lat + g.lat_rs[l + 1] + bb)) {
          FdItem it{f, (uint32_t)(l + 1), (uint32_t)bb, 0};
          ctx.template emit<RESIZE>(&it);
        }
      }
    }
  }

  // Scan (round 2): per-warp cascade-stage lists.  A warp that runs 32 windows through
  // the cascade in lockstep pays for its deepest window: with ~30% of windows passing
  // stage 0 and a few near every face reaching stage 11, a warp almost always ran all 12
  // stages (~90 weak classifiers) while the mean window needs ~5.  Block-wide stage passes
  // (one barrier per stage) fixed the divergence but left most warps waiting at the
  // barriers of the sparse late stages (ncu: 58% of stall samples).  So each worker warp
  // owns a contiguous range of the batch's windows (the rows concatenated) and, in shared
  // memory, one list per stage s >= 1 of windows that passed stage s-1.  Every step
  // evaluates ONE stage for 32 windows: the deepest list holding >= 32 entries, else the
  // next 32 windows of the range (stage 0), else (range exhausted) the shallowest
  // non-empty list, partially.  A step adds <= 32 entries to the next list, which is then
  // the deepest full one and is drained next, so no list exceeds 63 entries.  No block
  // barrier, the weak classifiers of a step are warp-uniform (broadcast loads), and the
  // lanes idle only in the final partial steps.  List counts live lane-distributed in
  // registers (lane s: list s), as do the per-stage survivor counts.  The cascade is read
  // through the read-only path (a kernel parameter array), the LBP codes with plain
  // L1-cacheable loads -- they were written in this run, but every Scan item reached its
  // block through a ring slot acquired with ld.acquire.gpu after the producer's release
  // (DESIGN.md §4.9 coherence argument).  Entries are (row << 13) | x, hence W <= 8192.
  static constexpr int kListCap = 64, kListsPerWarp = 15;  // stages 1 .. 15
  static constexpr int kScanScratch = kThreads / 32 * kListsPerWarp * kListCap * 2;

  // one weak classifier of a window (win = its top-left LBP code, W = the row pitch):
  // the window's LBP code at (cx, cy) picks a bit of the 256-bit mask
  static __device__ __forceinline__ int32_t weak_vote(const int32_t* wk, const uint8_t* win, int W) {
    const uint32_t code = win[__ldg(wk + 1) * W + __ldg(wk)];
    const uint32_t bit = ((uint32_t)__ldg(wk + 2 + (code >> 5)) >> (code & 31u)) & 1u;
    return bit ? __ldg(wk + 10) : __ldg(wk + 11);
  }

  // A batch may exceed max_batch(SCAN): an RTC [.., Scan] chain runs all the block-local
  // Scan items of its LBP batch at once.  Rows are taken 8 at a time (every list drains
  // before the next group).
  template <class Ctx>
  static __device__ void scan_batch(Ctx& ctx, const FdItem* items, int n) {
    for (int r0 = 0; r0 < n; r0 += 8) scan_rows(ctx, items + r0, min(8, n - r0));
  }

  template <class Ctx>
  static __device__ void scan_rows(Ctx& ctx, const FdItem* items, int n) {
    const Params& p = ctx.params();
    const FdGeo g(p.W, p.H);
    const int lane = threadIdx.x & 31, wid = threadIdx.x >> 5;
    const unsigned lt = (1u << lane) - 1u;
    uint16_t* lists = (uint16_t*)ctx.scratch() + wid * kListsPerWarp * kListCap - kListCap;  // list s at s * kListCap
    // lane k < n: batch row k (its first window's LBP row, pitch, window count)
    const uint8_t* myrow = p.lbp;
    int myW = 0, mylen = 0;
    if (lane < n) {
      const FdItem it = items[lane];
      if (it.frame < (uint32_t)p.n_frames && (int)it.level < g.L) {
        myW = g.W[it.level];
        mylen = myW - kWin + 1;
        myrow = p.lbp + (size_t)it.frame * g.off[g.L] + g.off[it.level] + (size_t)it.a * myW;
      }
    }
    int incl = mylen;
#pragma unroll
    for (int o = 1; o < 8; o <<= 1) {
      const int v = __shfl_up_sync(0xffffffffu, incl, o);
      if (lane >= o) incl += v;
    }
    int start[9];  // start[k] = first window of row k (rows of the batch concatenated)
    start[0] = 0;
#pragma unroll
    for (int k = 0; k < 8; ++k) start[k + 1] = __shfl_sync(0xffffffffu, incl, k);
    const int total = start[8], K = p.n_stages;
    const int lo = (int)((long long)total * wid / (kThreads / 32));
    const int hi = (int)((long long)total * (wid + 1) / (kThreads / 32));
    // lane s < K: stage s's weak-classifier offset, count and threshold
    int woff = 0, nw = 0, thr = 0;
    if (lane < K) {
      for (int q = 0; q < lane; ++q) woff += p.n_weak[q];
      nw = p.n_weak[lane];
      thr = p.thr[lane];
    }
    int cnt = 0;                   // lane s in [1, K): entries in list s
    unsigned long long surv = 0;   // lane s < K: windows that passed stage s
    int next = lo;
    const bool list_lane = lane >= 1 && lane < K;
    for (;;) {
      int s, take;
      const unsigned full = __ballot_sync(0xffffffffu, list_lane && cnt >= 32);
      if (full) {
        s = 31 - __clz(full);
        take = 32;
      } else if (next < hi) {
        s = 0;
        take = min(32, hi - next);
      } else {
        const unsigned any = __ballot_sync(0xffffffffu, list_lane && cnt > 0);
        if (!any) break;
        s = __ffs(any) - 1;
        take = __shfl_sync(0xffffffffu, cnt, s);
      }
      const bool v = lane < take;
      int k = 0, x = 0;
      if (s == 0) {
        const int i = next + lane;
#pragma unroll
        for (int q = 1; q < 8; ++q) k += i >= start[q] ? 1 : 0;
        x = i - start[k];
        next += take;
      } else {
        const int c = __shfl_sync(0xffffffffu, cnt, s);
        if (v) {
          const uint32_t e = lists[s * kListCap + c - take + lane];
          k = (int)(e >> 13);
          x = (int)(e & 0x1fffu);
        }
        if (lane == s) cnt -= take;
      }
      if (!v) k = 0, x = 0;
      const unsigned long long rb = (unsigned long long)__shfl_sync(0xffffffffu, (unsigned long long)myrow, k);
      const int W = __shfl_sync(0xffffffffu, myW, k);
      const int so = __shfl_sync(0xffffffffu, woff, s), sn = __shfl_sync(0xffffffffu, nw, s);
      const int st = __shfl_sync(0xffffffffu, thr, s);
      int32_t sum = 0;
      if (v) {
        const uint8_t* win = (const uint8_t*)rb + x;
        const int32_t* wk = p.weak + 12 * so;
#pragma unroll 4
        for (int w = 0; w < sn; ++w, wk += 12) sum += weak_vote(wk, win, W);
      }
      const bool pass = v && sum >= st;
      const unsigned bm = __ballot_sync(0xffffffffu, pass);
      if (lane == s) surv += (unsigned long long)__popc(bm);
      if (bm) {
        if (s + 1 == K) {
          emit_dets(p, items, bm, pass, k, x);
        } else {
          const int c = __shfl_sync(0xffffffffu, cnt, s + 1);
          if (pass) lists[(s + 1) * kListCap + c + __popc(bm & lt)] = (uint16_t)((k << 13) | x);
          if (lane == s + 1) cnt += __popc(bm);
        }
      }
      __syncwarp();
    }
    if (lane < K && surv) atomicAdd(p.survivors + lane, surv);
    if (threadIdx.x == 0 && total) atomicAdd(p.windows, (unsigned long long)total);
  }

  // detections of the warp's passing lanes (mask bm): warp-aggregated append
  static __device__ __forceinline__ void emit_dets(const Params& p, const FdItem* items, unsigned bm, bool pass, int k, int x) {
    const int lane = threadIdx.x & 31, leader = __ffs(bm) - 1;
    unsigned long long base = 0;
    if (lane == leader) base = atomicAdd(p.det_count, (unsigned long long)__popc(bm));
    base = __shfl_sync(0xffffffffu, base, leader);
    if (pass) {
      const FdItem it = items[k];
      const unsigned long long di = base + __popc(bm & ((1u << lane) - 1u));
      if (di < p.det_cap) *(uint4*)(p.det + 4 * di) = make_uint4(it.frame, it.level, (uint32_t)x, it.a);
    }
  }

  template <int s, class Ctx>
  static __device__ void exec(Ctx& ctx, const uint8_t* items, int n) {
    if constexpr (s == SCAN) {
      scan_batch(ctx, (const FdItem*)items, n);
      return;
    }
    const Params& p = ctx.params();
    const FdGeo g(p.W, p.H);
    const size_t npx = (size_t)p.W * p.H;
    const int t = threadIdx.x;
    for (int k = 0; k < n; ++k) {
      const FdItem it = ((const FdItem*)items)[k];
      if (it.frame >= (uint32_t)p.n_frames) continue;
      const uint32_t f = it.frame;
      uint8_t* img = p.levels + (size_t)f * g.off[g.L];
      uint8_t* lbp = p.lbp + (size_t)f * g.off[g.L];
      const uint8_t* rgb = p.rgb + (size_t)f * npx * 3;
      if constexpr (s == GRAY) {
        uint32_t* hs = (uint32_t*)ctx.scratch();
        hs[t] = 0;
        worker_sync();
        const int y0 = (int)it.a * kBand, y1 = min(y0 + kBand, p.H);
        for (size_t q = (size_t)y0 * p.W + t; q < (size_t)y1 * p.W; q += kThreads) atomicAdd(&hs[fd_gray(rgb + 3 * q)], 1u);
        worker_sync();
        if (hs[t]) atomicAdd(&p.hist[(size_t)f * 256 + t], hs[t]);
        worker_sync();
        if (t == 0 && fd_latch(latches(p, g, f))) {
          FdItem c{f, 0, 0, 0};
          ctx.template emit<CDF>(&c);
        }
      } else if constexpr (s == CDF) {
        uint32_t* cs = (uint32_t*)ctx.scratch();
        __shared__ int first_s;
        const uint32_t h = __ldcg(&p.hist[(size_t)f * 256 + t]);
        cs[t] = h;
        if (t == 0) first_s = 256;
        worker_sync();
        for (int o = 1; o < 256; o <<= 1) {
          uint32_t v = t >= o ? cs[t - o] : 0u;
          worker_sync();
          cs[t] += v;
          worker_sync();
        }
        if (h != 0u) atomicMin(&first_s, t);
        worker_sync();
        const int fb = first_s;
        const unsigned long long N = npx, cmin = fb < 256 ? cs[fb] : 0ull;
        uint8_t v;
        if (N == cmin) v = (uint8_t)t;
        else if (t < fb) v = 0;
        else v = (uint8_t)((((unsigned long long)cs[t] - cmin) * 255ull + (N - cmin) / 2ull) / (N - cmin));
        p.lut[(size_t)f * 256 + t] = v;
        worker_sync();
        for (int b = t; b < g.nb[0]; b += kThreads) {
          FdItem m{f, 0, (uint32_t)b, 0};
          ctx.template emit<MAP>(&m);
        }
      } else if constexpr (s == MAP) {
        uint8_t* lut = ctx.scratch();
        lut[t] = __ldcg(p.lut + (size_t)f * 256 + t);
        worker_sync();
        const int y0 = (int)it.a * kBand, y1 = min(y0 + kBand, p.H);
        for (size_t q = (size_t)y0 * p.W + t; q < (size_t)y1 * p.W; q += kThreads) img[q] = lut[fd_gray(rgb + 3 * q)];
        worker_sync();
        if (t == 0) image_band_done(ctx, p, g, f, 0, (int)it.a);
      } else if constexpr (s == RESIZE) {
        const int l = (int)it.level;
        if (l < 1 || l >= g.L) continue;
        const uint8_t* src = img + g.off[l - 1];
        uint8_t* dst = img + g.off[l];
        const int W = g.W[l], Wp = g.W[l - 1];
        const int y0 = (int)it.a * kBand, y1 = min(y0 + kBand, g.H[l]);
        for (int q = t; q < (y1 - y0) * W; q += kThreads) {
          const int y = y0 + q / W, x = q % W;
          dst[(size_t)y * W + x] = __ldcg(src + (size_t)((5 * y) >> 2) * Wp + ((5 * x) >> 2));
        }
        worker_sync();
        if (t == 0) image_band_done(ctx, p, g, f, l, (int)it.a);
      } else if constexpr (s == LBP) {
        const int l = (int)it.level;
        if (l >= g.L) continue;
        const uint8_t* im = img + g.off[l];
        uint8_t* lb = lbp + g.off[l];
        const int W = g.W[l], H = g.H[l];
        const int y0 = (int)it.a * kBand, y1 = min(y0 + kBand, H);
        for (int q = t; q < (y1 - y0) * W; q += kThreads) {
          const int y = y0 + q / W, x = q % W;
          uint8_t code = 0;
          if (x > 0 && y > 0 && x < W - 1 && y < H - 1) {
            const uint8_t* c = im + (size_t)y * W + x;
            const uint8_t cv = __ldcg(c);
            code = (uint8_t)((__ldcg(c - W - 1) >= cv) | ((__ldcg(c - W) >= cv) << 1) | ((__ldcg(c - W + 1) >= cv) << 2) |
                             ((__ldcg(c + 1) >= cv) << 3) | ((__ldcg(c + W + 1) >= cv) << 4) |
                             ((__ldcg(c + W) >= cv) << 5) | ((__ldcg(c + W - 1) >= cv) << 6) | ((__ldcg(c - 1) >= cv) << 7));
          }
          lb[(size_t)y * W + x] = code;
        }
        worker_sync();
        if (t < 2) {  // window-row groups g = band-1 (t == 0) and band (t == 1)
          const int gr = (int)it.a - 1 + t;
          if (gr >= 0 && gr * kBand <= H - kWin && fd_latch(latches(p, g, f) + g.lat_scan[l] + gr)) {
            const int ylast = min(gr * kBand + kBand - 1, H - kWin);
            for (int y = gr * kBand; y <= ylast; ++y) {
              FdItem sc{f, (uint32_t)l, (uint32_t)y, 0};
              ctx.template emit<SCAN>(&sc);
            }
          }
        }
      }
      worker_sync();
    }
  }

  static cudaError_t init_run(const Params& p, cudaStream_t st);
  static cudaError_t finalize(const Params&, cudaStream_t) { return cudaSuccess; }
  static bool output(const Params& p, int idx, void** ptr, size_t* bytes) {
    if (idx == 0) { *ptr = p.det; *bytes = 16 * (size_t)p.det_cap; return true; }
    if (idx == 1) { *ptr = p.det_count; *bytes = 8; return true; }
    return false;
  }
  static const char* validate(const Params& p) {
    if (p.W < kWin || p.H < kWin || p.H > kMaxBands0 * kBand || p.W > 8192)
      return "vp_facedet_params: 24 <= W <= 8192, 24 <= H <= 2048";
    if (p.n_frames <= 0 || p.n_stages <= 0 || p.n_stages > 16) return "vp_facedet_params: bad n_frames / n_stages";
    int tot = 0;
    for (int k = 0; k < p.n_stages; ++k) tot += p.n_weak[k];
    if (tot != p.n_weak_total || tot * 12 * 4 > 6144) return "vp_facedet_params: n_weak_total must be sum(n_weak) <= 128";
    if (!p.rgb || !p.levels || !p.lbp || !p.hist || !p.lut || !p.weak || !p.det || !p.det_count || !p.survivors ||
        !p.windows || !p.latch)
      return "vp_facedet_params: all buffers are required";
    if ((uintptr_t)p.det & 15) return "vp_facedet_params: det must be 16-B aligned";
    return nullptr;
  }
};

__global__ void k_fd_init(vp_facedet_params p) {
  const FdGeo g(p.W, p.H);
  const size_t tot = g.lat_per * (size_t)p.n_frames;
  for (size_t i = blockIdx.x * (size_t)blockDim.x + threadIdx.x; i < tot; i += (size_t)gridDim.x * blockDim.x) {
    const size_t k = i % g.lat_per;
    int v = 0;
    if (k == 0) {
      v = g.nb[0];
    } else {
      for (int l = 0; l < g.L; ++l) {
        if (k >= g.lat_rs[l] && k < g.lat_rs[l] + g.nb[l]) {
          const int b = (int)(k - g.lat_rs[l]);
          int s0 = 0, s1 = 0;
          if (l > 0) g.resize_src(l, b, s0, s1);
          v = l > 0 ? s1 - s0 + 1 : 0;
        } else if (k >= g.lat_lbp[l] && k < g.lat_lbp[l] + g.nb[l]) {
          const int b = (int)(k - g.lat_lbp[l]);
          v = (b > 0) + 1 + (b + 1 < g.nb[l]);
        } else if (k >= g.lat_scan[l] && k < g.lat_scan[l] + g.nb[l]) {
          const int b = (int)(k - g.lat_scan[l]);
          v = 1 + (b + 1 < g.nb[l]);
        }
      }
    }
    p.latch[i] = v;
  }
  for (size_t i = blockIdx.x * (size_t)blockDim.x + threadIdx.x; i < 256 * (size_t)p.n_frames;
       i += (size_t)gridDim.x * blockDim.x)
    p.hist[i] = 0;
  if (blockIdx.x == 0 && threadIdx.x < 16) p.survivors[threadIdx.x] = 0;
  if (blockIdx.x == 0 && threadIdx.x == 0) {
    *p.det_count = 0;
    *p.windows = 0;
  }
}

cudaError_t FaceDetF::init_run(const Params& p, cudaStream_t st) {
  k_fd_init<<<148, 256, 0, st>>>(p);
  return cudaGetLastError();
}

const FamilyOps* family_facedet() {
  static FamilyImpl<FaceDetF> f("facedet");
  return &f;
}

}  // namespace vp

// fam_reyes.cu — Reyes rendering as VersaPipe stages (Fig. 1: Primitives ->
// Bound -> diceable? -> Split (back to Bound) | Dice -> Shade -> Image; L55; Table 2 272-B
// item).  The paper gives no formulas; the arithmetic follows DESIGN.md §2 readings
// R-R1..R-R12.  Compiled with -fmad=false: every float operation is a
// separately rounded IEEE op in the written order, so results are bit-identical to the
// CPU oracle.
//
// Thread mapping (threadNum, L37): Bound 16 threads/patch (one per control point),
// Split 16 (one per output control point), Dice 32 (one warp per patch, 81 grid points),
// Shade 64 (one per micropolygon).
#include <math.h>

#include <limits.h>

#include <algorithm>

#include "../../include/vp.h"
#include "vp_family.cuh"

namespace vp {

#ifndef VP_REYES_MINB
#define VP_REYES_MINB 3
#endif
#ifndef VP_DS_MINB          // resident blocks/SM the RTC [Dice, Shade] kernel is built for
#define VP_DS_MINB 3
#endif
#ifndef VP_DS_BATCH         // its Dice batch (staging: 2 x batch x 208 B per block)
#define VP_DS_BATCH 64
#endif
#ifndef VP_BS_MINB          // resident blocks/SM the block-local [Bound, Split] kernel is built for
#define VP_BS_MINB 4
#endif

// Patch item as queued, 208 B (reading R-S10): the paper's 272-B item (Table 2:
// float4 control points) carries w = 1 in every point -- the patches are polynomial
// (affine control points) and de Casteljau keeps w = (1 + 1) / 2 = 1 exactly -- so the
// queues carry x, y, z only, as three 16-float planes (§8.5: "methods that
// reduce data item size in the queues could also be beneficial").  P[a][b] is point
// 4a + b (a = u index, b = v index).
struct RPatch {
  float x[16], y[16], z[16];
  uint32_t id, path, dirs, depth;
};
static_assert(sizeof(RPatch) == 208, "queued patch item is 208 B");

// control point k as (x, y, z, w = 1) / its x, y, z into a patch
__device__ __forceinline__ float4 cp_get(const RPatch* P, int k) { return make_float4(P->x[k], P->y[k], P->z[k], 1.0f); }
__device__ __forceinline__ void cp_put(RPatch* P, int k, const float4 v) {
  P->x[k] = v.x;
  P->y[k] = v.y;
  P->z[k] = v.z;
}

constexpr int kG = 8, kNG = 9, kNP = 81;
// Dice -> Shade item (2032 B).  Grid point (i, j) = S(i/8, j/8) is o[9j + i] (v-major: Dice's
// lanes then take consecutive points of one u-curve row, so the 4 u-curve points each reads
// are the same for 9 lanes -- shared-memory broadcasts instead of bank conflicts) and
// s[10j + i] (a padded row: the 16 lanes of a 64-bit load phase of the box test, (i, j) and
// (i + 1, j) for j = 0..7, then hit 16 distinct bank pairs).  o = object-space point
// (x, y, z) with its screen depth zs in .w, so Shade's normal and depth take 4 16-B loads;
// s = the Q8 fixed-point snap of (sx, sy) (reading R-R9; INT_MIN where it does not fit).  While Dice runs, s[] stages the
// 36 u-curve points C_a(v_j) as float4.  (Round 2: carrying each point's pixel-centre
// index range as well -- a 2608-B grid -- made the box test cheaper but pushed the fused
// kernel's shared memory past the 196-KB carve-out step, and it ran 5% slower.)
#ifndef VP_MS_REG  // 1: Dice keeps the frame matrix rows in registers for a lane's 3 points
#define VP_MS_REG 1
#endif
#ifndef VP_SROW
#define VP_SROW 10
#endif
constexpr int kSR = VP_SROW;  // row stride of RGrid::s (9: unpadded)
__device__ __forceinline__ int sidx(int i, int j) { return j * kSR + i; }
struct RGrid {
  uint32_t id, path, depth, dirs;
  float4 o[kNP];
  int2 s[kSR * kG + kNG];
};
static_assert(sizeof(RGrid) == (kSR == 10 ? 2032 : 1968), "grid item stride");
static_assert(sizeof(int2) * kNP >= sizeof(float4) * 4 * kNG, "u-curve staging fits in s[]");

struct __align__(16) FbRec {
  unsigned long long key;
  float s;
  uint32_t pad;
};

__device__ __forceinline__ float4 project(const float* __restrict__ M, float x, float y, float z, float w) {
  float c[4];
#pragma unroll
  for (int r = 0; r < 4; ++r) {
    float acc = __ldg(M + 4 * r + 0) * x;
    acc = acc + __ldg(M + 4 * r + 1) * y;
    acc = acc + __ldg(M + 4 * r + 2) * z;
    acc = acc + __ldg(M + 4 * r + 3) * w;
    c[r] = acc;
  }
  return make_float4(c[0], c[1], c[2], c[3]);
}

__device__ __forceinline__ void screen(const vp_reyes_params& p, float4 c, float& sx, float& sy, float& zs) {
  float nx = c.x / c.w;
  float ny = c.y / c.w;
  sx = (nx * 0.5f + 0.5f) * (float)p.W;
  sy = (ny * 0.5f + 0.5f) * (float)p.H;
  zs = c.z / c.w;
}

__device__ __forceinline__ float red16_max(float v) {
#pragma unroll
  for (int o = 8; o >= 1; o >>= 1) v = fmaxf(v, __shfl_xor_sync(0xffffffffu, v, o, 16));
  return v;
}
__device__ __forceinline__ float red16_min(float v) {
#pragma unroll
  for (int o = 8; o >= 1; o >>= 1) v = fminf(v, __shfl_xor_sync(0xffffffffu, v, o, 16));
  return v;
}

__device__ __forceinline__ void bernstein(float t, float B[4]) {
  float s = 1.0f - t;
  B[0] = (s * s) * s;
  B[1] = ((3.0f * t) * s) * s;
  B[2] = ((3.0f * t) * t) * s;
  B[3] = (t * t) * t;
}

__device__ __forceinline__ uint32_t zkey(float z) {
  uint32_t b = __float_as_uint(z);
  return (b & 0x80000000u) ? ~b : (b | 0x80000000u);
}

template <class I>
__device__ __forceinline__ I edge(I ax, I ay, I bx, I by, I px, I py) {
  return (bx - ax) * (py - ay) - (by - ay) * (px - ax);
}
// top-left-style ownership of boundary points (reading R-R9)
template <class I>
__device__ __forceinline__ bool owns(I ax, I ay, I bx, I by) {
  I dx = bx - ax, dy = by - ay;
  return dy > 0 || (dy == 0 && dx < 0);
}
__device__ __forceinline__ long long fdiv256(long long a) { return a >> 8; }  // floor(a / 256)

// 128-bit compare-and-swap (sm_90+): atomically keep the minimum key with its shade factor.
__device__ __forceinline__ void fb_min(FbRec* rec, unsigned long long key, float s) {
  unsigned long long* a = (unsigned long long*)rec;
  // first attempt assumes the cleared record {UINT64_MAX, 0}: one L2 round trip for a
  // first touch; otherwise the failed CAS returns the current record
  unsigned long long cur_k = ~0ull, cur_s = 0ull;
  const unsigned long long new_s = (unsigned long long)__float_as_uint(s);
  while (key < cur_k) {
    unsigned long long ok, os;
    asm volatile(
        "{\n\t.reg .b128 c, n, o;\n\t"
        "mov.b128 c, {%2, %3};\n\t"
        "mov.b128 n, {%4, %5};\n\t"
        "atom.global.relaxed.gpu.cas.b128 o, [%6], c, n;\n\t"
        "mov.b128 {%0, %1}, o;\n\t}"
        : "=l"(ok), "=l"(os)
        : "l"(cur_k), "l"(cur_s), "l"(key), "l"(new_s), "l"(a)
        : "memory");
    if (ok == cur_k && os == cur_s) return;
    cur_k = ok;
    cur_s = os;
  }
}

// Pixel-centre loop of one positively oriented triangle, coordinates relative to an
// origin inside its bounding box (exact in I: int32 when the box is < 2^14 Q8 units).
template <class I>
__device__ __forceinline__ void cover(const vp_reyes_params& p, FbRec* fb, I ax, I ay, I bx, I by, I cx, I cy,
                                      long long ox, long long oy, long long px0, long long px1, long long py0,
                                      long long py1, unsigned long long key, float s) {
  const bool o0 = owns(ax, ay, bx, by), o1 = owns(bx, by, cx, cy), o2 = owns(cx, cy, ax, ay);
  for (long long py = py0; py <= py1; ++py) {
    const I Y = (I)(py * 256 + 128 - oy);
    for (long long px = px0; px <= px1; ++px) {
      const I X = (I)(px * 256 + 128 - ox);
      I w0 = edge(ax, ay, bx, by, X, Y), w1 = edge(bx, by, cx, cy, X, Y), w2 = edge(cx, cy, ax, ay, X, Y);
      bool in = (w0 > 0 || (w0 == 0 && o0)) && (w1 > 0 || (w1 == 0 && o1)) && (w2 > 0 || (w2 == 0 && o2));
      if (in) fb_min(fb + (size_t)py * p.W + px, key, s);
    }
  }
}

// One triangle of a micropolygon in the int32 quad path: three edge functions biased so
// that "inside or owned boundary" (reading R-R9) is w >= 0, evaluated incrementally
// along a pixel row (exact integer arithmetic, so identical to a direct evaluation).
struct TriEdges {
  int w[3], dx[3], dy[3];  // w at the row-start sample; per-pixel-step and per-row-step increments
  bool live;
};
__device__ __forceinline__ void tri_setup(TriEdges& T, int ax, int ay, int bx, int by, int cx, int cy, int X0, int Y0) {
  const int area = edge(ax, ay, bx, by, cx, cy);
  T.live = area != 0;
  if (area < 0) {  // positive orientation: (a, c, b)
    int tx = bx, ty = by;
    bx = cx; by = cy; cx = tx; cy = ty;
  }
  const int ex[3] = {ax, bx, cx}, ey[3] = {ay, by, cy};
#pragma unroll
  for (int k = 0; k < 3; ++k) {
    const int px = ex[k], py = ey[k], qx = ex[(k + 1) % 3], qy = ey[(k + 1) % 3];
    const int bias = owns(px, py, qx, qy) ? 0 : -1;
    T.w[k] = edge(px, py, qx, qy, X0, Y0) + bias;
    T.dx[k] = -(qy - py) * 256;
    T.dy[k] = (qx - px) * 256;
  }
}

__device__ void raster_tri(const vp_reyes_params& p, FbRec* fb, long long ax, long long ay, long long bx, long long by,
                           long long cx, long long cy, unsigned long long key, float s) {
  long long xmin = min(ax, min(bx, cx)), xmax = max(ax, max(bx, cx));
  long long ymin = min(ay, min(by, cy)), ymax = max(ay, max(by, cy));
  long long px0 = -fdiv256(-(xmin - 128)), px1 = fdiv256(xmax - 128);
  long long py0 = -fdiv256(-(ymin - 128)), py1 = fdiv256(ymax - 128);
  if (px0 < 0) px0 = 0;
  if (py0 < 0) py0 = 0;
  if (px1 > p.W - 1) px1 = p.W - 1;
  if (py1 > p.H - 1) py1 = p.H - 1;
  if (px0 > px1 || py0 > py1) return;  // no pixel centre inside the box
  if (xmax - xmin < (1ll << 14) && ymax - ymin < (1ll << 14)) {
    // every |difference| < 2^14 -> products < 2^28: int32 is exact
    int Ax = (int)(ax - xmin), Ay = (int)(ay - ymin), Bx = (int)(bx - xmin), By = (int)(by - ymin);
    int Cx = (int)(cx - xmin), Cy = (int)(cy - ymin);
    int area = edge(Ax, Ay, Bx, By, Cx, Cy);
    if (area == 0) return;
    if (area < 0) cover<int>(p, fb, Ax, Ay, Cx, Cy, Bx, By, xmin, ymin, px0, px1, py0, py1, key, s);
    else cover<int>(p, fb, Ax, Ay, Bx, By, Cx, Cy, xmin, ymin, px0, px1, py0, py1, key, s);
  } else {
    long long area = edge(ax, ay, bx, by, cx, cy);
    if (area == 0) return;
    if (area < 0) cover<long long>(p, fb, ax, ay, cx, cy, bx, by, 0, 0, px0, px1, py0, py1, key, s);
    else cover<long long>(p, fb, ax, ay, bx, by, cx, cy, 0, 0, px0, px1, py0, py1, key, s);
  }
}

// Scratch of the fused [Dice, Shade] chain.
struct ChainScratch {
  float4 M[kWarpsW][2][4];     // per-warp copies of the pair's frame matrices (rows)
  float B[kWarpsW][36];        // per-warp Bernstein table B_b(j/8), [9][4]
  uint8_t list[kWarpsW][128];  // per-warp compacted list of pixel-covering micropolygons (q | grid << 6)
};

struct ReyesF {
  static constexpr int S = 4;
  static constexpr int BOUND = 0, SPLIT = 1, DICE = 2, SHADE = 3;
  static constexpr int kinds[S] = {VP_REYES_BOUND, VP_REYES_SPLIT, VP_REYES_DICE, VP_REYES_SHADE};
  using Params = vp_reyes_params;
  static constexpr int stride(int s) { return s == SHADE ? (int)sizeof(RGrid) : (int)sizeof(RPatch); }
  static constexpr int threads_per_item(int s) { return s == BOUND ? 16 : s == SPLIT ? 16 : s == DICE ? 32 : 64; }
  static constexpr int max_batch(int s) { return s == BOUND ? 32 : s == SPLIT ? 16 : s == DICE ? 64 : 4; }
  // Dice batches above 8 only where the fused [Dice, Shade] chain runs them (grids in one
  // block-local slot per warp): the RTC kernel (64) and a megakernel with depth-first
  // [Bound, Split] (32: the in buffers stay at the Bound batch's size); elsewhere every
  // diced grid needs an out-buffer slot.
  static constexpr int kernel_max_batch(int lo, int hi, bool rtc, int s) {
    // depth-first [Bound, Split] (exec_dfs): 32 seeds per claim, two per 16-thread group
    if (!rtc && lo == BOUND && hi >= SPLIT && (s == BOUND || s == SPLIT)) return s == BOUND ? 32 : 16;  // DFS kernels
    if (s == DICE && !rtc && lo == BOUND && hi == SHADE) return 32;
    if (s == DICE && rtc && lo == DICE && hi == SHADE) return VP_DS_BATCH;
    return (s == DICE && !(rtc && lo == DICE && hi == SHADE)) ? 8 : max_batch(s);
  }
  static constexpr int fused_local_cap(int, int, int) { return kThreads / 32; }
  static constexpr int default_batch(int s) { return max_batch(s); }
  static constexpr int fanout(int s, int t) {
    return (s == BOUND && (t == SPLIT || t == DICE)) ? 1 : (s == SPLIT && t == BOUND) ? 2 : (s == DICE && t == SHADE) ? 1 : 0;
  }
  static constexpr bool rtc_ok(int, int) { return true; }
  // every kernel whose range ends in [Dice, Shade] may run the fused chain (an RTC
  // kernel [Split..Shade] fuses its Dice batches too), so each reserves the chain scratch
  static constexpr int scratch_bytes(int lo, int hi) { return scratch_bytes_k(lo, hi, true); }
  // the fused [Dice, Shade] chain runs only in RTC kernels; block-local recursion only in
  // non-RTC ones (a megakernel [Bound..Shade] must not pay for the chain's scratch: it sits
  // at the edge of 2 blocks per SM)
  static constexpr int scratch_bytes_k(int lo, int hi, bool rtc) {
    return (((rtc || local_recursion(lo, hi)) && lo <= DICE && hi == SHADE) ? (int)sizeof(ChainScratch) : 0) +
           ((!rtc && lo == BOUND && hi >= SPLIT) ? (int)((sizeof(DfsScratch) + 127) / 128 * 128) : 0);
  }
  static constexpr int default_cap_log2(int s) { return s == BOUND ? 20 : s == SHADE ? 17 : 19; }
  // register budget: kernels containing Shade are held to 3 resident blocks per SM
  static constexpr int min_blocks(int lo, int hi, bool rtc) {
    return (!rtc && lo == BOUND && hi == SPLIT) ? VP_BS_MINB : (rtc && lo == DICE && hi == SHADE) ? VP_DS_MINB : VP_REYES_MINB;
  }

  template <int s>
  static __device__ unsigned long long item_id(const uint8_t* it) {
    // node id = (id << 12) | (depth << 8) | path  (frame, patch, depth, path)
    if constexpr (s == SHADE) {
      const RGrid* g = (const RGrid*)it;
      return ((unsigned long long)g->id << 12) | ((unsigned long long)(g->depth & 15u) << 8) | (g->path & 0xFFu);
    } else {
      const RPatch* q = (const RPatch*)it;
      return ((unsigned long long)q->id << 12) | ((unsigned long long)(q->depth & 15u) << 8) | (q->path & 0xFFu);
    }
  }

  template <int s, class Ctx>
  static __device__ void exec(Ctx& ctx, const uint8_t* items, int n) {
    if constexpr (s == BOUND) bound(ctx, items, n);
    else if constexpr (s == SPLIT) split(ctx, items, n);
    else if constexpr (s == DICE) dice(ctx, items, n);
    else shade(ctx, items, n);
  }

  // -------------------------------------------------------------- Bound (16 thr/patch)
  // Bound of patch P by one 16-thread group (lane = its control point; both groups of a
  // warp call together, `valid` may differ): returns 0 cull, 1 split, 2 dice (readings
  // R-R2..R-R5), the split direction, and this thread's control point q.
  // Mc / mframe: a shared-memory copy of one frame's matrix (block-local recursion: the
  // patches of a batch and their children almost always share the frame)
  static __device__ __forceinline__ int bound_patch(const Params& p, const RPatch* P, int lane, bool valid, int& dir,
                                                    float4& q, const float4* Mc = nullptr, uint32_t mframe = ~0u) {
    uint32_t frame = frame_of(p, P->id);
    q = cp_get(P, lane);
    return bound_q(p, q, P->depth, frame, lane, valid, dir, Mc, mframe);
  }
  // local frame index of an item id (frame << 12 | patch) in this run's matrices
  static __device__ __forceinline__ uint32_t frame_of(const Params& p, uint32_t id) {
    uint32_t frame = (id >> 12) - (uint32_t)p.frame_base;
    return frame >= (uint32_t)p.n_frames ? 0u : frame;
  }
  // Bound on a patch held in registers (lane = control point q of a 16-thread group).
  static __device__ __forceinline__ int bound_q(const Params& p, const float4 q, uint32_t depth, uint32_t frame,
                                                int lane, bool valid, int& dir, const float4* Mc, uint32_t mframe) {
    const float* M = p.M + 16 * (size_t)frame;
    float4 c;
    if (Mc && frame == mframe) {
      float cc[4];
#pragma unroll
      for (int r = 0; r < 4; ++r) {  // project() with the rows from shared memory (same op order)
        const float4 m = Mc[r];
        float acc = m.x * q.x;
        acc = acc + m.y * q.y;
        acc = acc + m.z * q.z;
        acc = acc + m.w;  // m.w * q.w with q.w = 1 exactly (R-S10): x * 1 = x in IEEE arithmetic
        cc[r] = acc;
      }
      c = make_float4(cc[0], cc[1], cc[2], cc[3]);
    } else {
      c = project(M, q.x, q.y, q.z, q.w);
    }
    const bool behind = !(c.w > p.near_w);
    const unsigned bal = __ballot_sync(0xffffffffu, behind);
    const int nbehind = __popc((bal >> (threadIdx.x & 16)) & 0xFFFFu);
    float sx, sy, zs;
    screen(p, c, sx, sy, zs);
    const float xmin = red16_min(sx), xmax = red16_max(sx), ymin = red16_min(sy), ymax = red16_max(sy);
    // The split metrics are computed only where a split needs them (the branch is uniform
    // per 16-thread group; the group's shuffles use its own half-warp mask).  max over
    // non-negative values is exact in any order, so the results equal a full evaluation.
    const unsigned gm = 0xFFFFu << (threadIdx.x & 16);
    int cls;  // 0 cull, 1 split, 2 dice
    dir = 0;
    if (!valid || nbehind == 16) {
      cls = 0;
    } else if (nbehind > 0) {
      cls = ((int)depth >= p.max_depth) ? 0 : 1;
      if (cls == 1) {  // object-space metric (near-plane straddle, R-R4)
        const float ox12 = __shfl_sync(gm, q.x, (lane & 3) + 12, 16), oy12 = __shfl_sync(gm, q.y, (lane & 3) + 12, 16),
                    oz12 = __shfl_sync(gm, q.z, (lane & 3) + 12, 16);
        const float ox3 = __shfl_down_sync(gm, q.x, 3, 16), oy3 = __shfl_down_sync(gm, q.y, 3, 16),
                    oz3 = __shfl_down_sync(gm, q.z, 3, 16);
        float olu = 0.0f, olv = 0.0f;
        if (lane < 4) {
          olu = fabsf(ox12 - q.x) + fabsf(oy12 - q.y);
          olu = olu + fabsf(oz12 - q.z);
        }
        if ((lane & 3) == 0) {
          olv = fabsf(ox3 - q.x) + fabsf(oy3 - q.y);
          olv = olv + fabsf(oz3 - q.z);
        }
#pragma unroll
        for (int o = 8; o >= 1; o >>= 1) {
          olu = fmaxf(olu, __shfl_xor_sync(gm, olu, o, 16));
          olv = fmaxf(olv, __shfl_xor_sync(gm, olv, o, 16));
        }
        dir = (olu >= olv) ? 0 : 1;
      }
    } else if (xmax < 0.0f || xmin >= (float)p.W || ymax < 0.0f || ymin >= (float)p.H) {
      cls = 0;
    } else {
      const float bw = xmax - xmin, bh = ymax - ymin;
      const float ext = bw > bh ? bw : bh;
      if ((int)depth >= p.max_depth || ext <= p.t_dice) {
        cls = 2;
      } else {  // screen-space split metric (reading R-R5)
        cls = 1;
        const float sx12 = __shfl_sync(gm, sx, (lane & 3) + 12, 16), sy12 = __shfl_sync(gm, sy, (lane & 3) + 12, 16);
        const float sx3 = __shfl_down_sync(gm, sx, 3, 16), sy3 = __shfl_down_sync(gm, sy, 3, 16);
        float lu = (lane < 4) ? fabsf(sx12 - sx) + fabsf(sy12 - sy) : 0.0f;
        float lv = ((lane & 3) == 0) ? fabsf(sx3 - sx) + fabsf(sy3 - sy) : 0.0f;
#pragma unroll
        for (int o = 8; o >= 1; o >>= 1) {
          lu = fmaxf(lu, __shfl_xor_sync(gm, lu, o, 16));
          lv = fmaxf(lv, __shfl_xor_sync(gm, lv, o, 16));
        }
        dir = (lu >= lv) ? 0 : 1;
      }
    }
    return cls;
  }

  // Bound for both 16-thread groups of a warp at once (all 32 lanes call it, converged;
  // `valid` may differ per group), the rows of each group's frame matrix in Mr: the same
  // operations as bound_q, with the split metrics' shuffles issued warp-uniformly (only
  // when some group of the warp needs them, never under divergence).
  static __device__ __forceinline__ int bound_warp(const Params& p, const float4 q, uint32_t depth, int lane,
                                                   bool valid, int& dir, const float4* Mr) {
    float cc[4];
#pragma unroll
    for (int r = 0; r < 4; ++r) {  // project() with the rows from shared memory (same op order)
      const float4 m = Mr[r];
      float acc = m.x * q.x;
      acc = acc + m.y * q.y;
      acc = acc + m.z * q.z;
      acc = acc + m.w;  // m.w * q.w with q.w = 1 exactly (R-S10): x * 1 = x in IEEE arithmetic
      cc[r] = acc;
    }
    const float4 c = make_float4(cc[0], cc[1], cc[2], cc[3]);
    const bool behind = !(c.w > p.near_w);
    const unsigned bal = __ballot_sync(0xffffffffu, behind);
    const int nbehind = __popc((bal >> (threadIdx.x & 16)) & 0xFFFFu);
    float sx, sy, zs;
    screen(p, c, sx, sy, zs);
    const float xmin = red16_min(sx), xmax = red16_max(sx), ymin = red16_min(sy), ymax = red16_max(sy);
    const bool deep = (int)depth >= p.max_depth;
    int cls;  // 0 cull, 1 split, 2 dice
    if (!valid || nbehind == 16) {
      cls = 0;
    } else if (nbehind > 0) {
      cls = deep ? 0 : 1;
    } else if (xmax < 0.0f || xmin >= (float)p.W || ymax < 0.0f || ymin >= (float)p.H) {
      cls = 0;
    } else {
      const float bw = xmax - xmin, bh = ymax - ymin;
      const float ext = bw > bh ? bw : bh;
      cls = (deep || ext <= p.t_dice) ? 2 : 1;
    }
    const bool straddle = nbehind > 0;
    dir = 0;
    // max over non-negative values is exact in any order: the results equal bound_q's
    if (__any_sync(0xffffffffu, cls == 1 && !straddle)) {  // screen-space split metric (R-R5)
      const float sx12 = __shfl_sync(0xffffffffu, sx, (lane & 3) + 12, 16);
      const float sy12 = __shfl_sync(0xffffffffu, sy, (lane & 3) + 12, 16);
      const float sx3 = __shfl_down_sync(0xffffffffu, sx, 3, 16), sy3 = __shfl_down_sync(0xffffffffu, sy, 3, 16);
      float lu = (lane < 4) ? fabsf(sx12 - sx) + fabsf(sy12 - sy) : 0.0f;
      float lv = ((lane & 3) == 0) ? fabsf(sx3 - sx) + fabsf(sy3 - sy) : 0.0f;
      // lu lives on the group's lanes 0..3, lv on lanes 0, 4, 8, 12: two levels each bring
      // both maxima to the group's lane 0, which decides for the group
      lu = fmaxf(lu, __shfl_xor_sync(0xffffffffu, lu, 1, 16));
      lu = fmaxf(lu, __shfl_xor_sync(0xffffffffu, lu, 2, 16));
      lv = fmaxf(lv, __shfl_xor_sync(0xffffffffu, lv, 4, 16));
      lv = fmaxf(lv, __shfl_xor_sync(0xffffffffu, lv, 8, 16));
      const int d0 = __shfl_sync(0xffffffffu, (lu >= lv) ? 0 : 1, 0, 16);
      if (!straddle) dir = d0;
    }
    if (__any_sync(0xffffffffu, cls == 1 && straddle)) {  // object-space metric (near-plane straddle, R-R4)
      const float ox12 = __shfl_sync(0xffffffffu, q.x, (lane & 3) + 12, 16);
      const float oy12 = __shfl_sync(0xffffffffu, q.y, (lane & 3) + 12, 16);
      const float oz12 = __shfl_sync(0xffffffffu, q.z, (lane & 3) + 12, 16);
      const float ox3 = __shfl_down_sync(0xffffffffu, q.x, 3, 16), oy3 = __shfl_down_sync(0xffffffffu, q.y, 3, 16),
                  oz3 = __shfl_down_sync(0xffffffffu, q.z, 3, 16);
      float olu = 0.0f, olv = 0.0f;
      if (lane < 4) {
        olu = fabsf(ox12 - q.x) + fabsf(oy12 - q.y);
        olu = olu + fabsf(oz12 - q.z);
      }
      if ((lane & 3) == 0) {
        olv = fabsf(ox3 - q.x) + fabsf(oy3 - q.y);
        olv = olv + fabsf(oz3 - q.z);
      }
      olu = fmaxf(olu, __shfl_xor_sync(0xffffffffu, olu, 1, 16));
      olu = fmaxf(olu, __shfl_xor_sync(0xffffffffu, olu, 2, 16));
      olv = fmaxf(olv, __shfl_xor_sync(0xffffffffu, olv, 4, 16));
      olv = fmaxf(olv, __shfl_xor_sync(0xffffffffu, olv, 8, 16));
      const int d0 = __shfl_sync(0xffffffffu, (olu >= olv) ? 0 : 1, 0, 16);
      if (straddle) dir = d0;
    }
    return cls;
  }

  template <class Ctx>
  static __device__ void bound(Ctx& ctx, const uint8_t* items, int n) {
    const Params& p = ctx.params();
    const int lane = threadIdx.x & 15;
    for (int r0 = 0; r0 < n; r0 += kThreads / 16) {
      const int k = r0 + (threadIdx.x >> 4);
      const bool valid = k < n;
      const RPatch* P = (const RPatch*)(items + (size_t)(valid ? k : 0) * sizeof(RPatch));
      int dir;
      float4 q;
      const int cls = bound_patch(p, P, lane, valid, dir, q);
      const uint32_t depth = P->depth;
      int slot = -1;
      if (lane == 0 && cls == 1) slot = ctx.template reserve<SPLIT>();
      if (lane == 0 && cls == 2) slot = ctx.template reserve<DICE>();
      slot = __shfl_sync(0xffffffffu, slot, 0, 16);
      if (cls != 0 && slot >= 0) {
        RPatch* out = (RPatch*)(cls == 1 ? ctx.template out_ptr<SPLIT>(slot) : ctx.template out_ptr<DICE>(slot));
        cp_put(out, lane, q);
        if (lane == 0) {
          out->id = P->id;
          out->path = P->path;
          out->dirs = (cls == 1) ? ((P->dirs & ~(1u << depth)) | ((uint32_t)dir << depth)) : P->dirs;
          out->depth = depth;
        }
      }
    }
  }

  // -------------------------------------------------------------- Split (16 thr/patch)
  // de Casteljau at t = 1/2 (reading R-R6) of the curve through this thread's control point
  // (thread `lane` of a 16-thread group): L / R are child control point `my` of the two halves.
  static __device__ __forceinline__ void split_cp(const RPatch* P, int dir, int lane, float4& L, float4& R, int& my) {
    const int line = lane >> 2, t = lane & 3;
    // control point u of this thread's curve: (u, line) for a u-split, (line, u) for v
    const int base = dir == 0 ? line : 4 * line, step = dir == 0 ? 4 : 1;
    my = base + step * t;
    const float4 a = cp_get(P, base), b = cp_get(P, base + step), c = cp_get(P, base + 2 * step),
                 d = cp_get(P, base + 3 * step);
    // per component, exactly this order
#define VP_CASTELJAU(comp)                                                   \
  {                                                                          \
    float ab = (a.comp + b.comp) * 0.5f, bc = (b.comp + c.comp) * 0.5f;      \
    float cd = (c.comp + d.comp) * 0.5f;                                     \
    float abc = (ab + bc) * 0.5f, bcd = (bc + cd) * 0.5f;                    \
    float m = (abc + bcd) * 0.5f;                                            \
    L.comp = t == 0 ? a.comp : t == 1 ? ab : t == 2 ? abc : m;              \
    R.comp = t == 0 ? m : t == 1 ? bcd : t == 2 ? cd : d.comp;              \
  }
    VP_CASTELJAU(x) VP_CASTELJAU(y) VP_CASTELJAU(z)  // w stays 1 (R-S10)
#undef VP_CASTELJAU
    L.w = R.w = 1.0f;
  }
  // children headers (split tree: path bit `depth` = 0 left / 1 right, dirs bit = direction)
  static __device__ __forceinline__ void split_headers(RPatch* l, RPatch* r, uint32_t id, uint32_t path, uint32_t dirs,
                                                       uint32_t depth, int dir) {
    l->id = r->id = id;
    l->dirs = r->dirs = (dirs & ~(1u << depth)) | ((uint32_t)dir << depth);
    l->depth = r->depth = depth + 1;
    l->path = path & ~(1u << depth);
    r->path = path | (1u << depth);
  }

  template <class Ctx>
  static __device__ void split(Ctx& ctx, const uint8_t* items, int n) {
    const int lane = threadIdx.x & 15;
    for (int r0 = 0; r0 < n; r0 += kThreads / 16) {
      const int k = r0 + (threadIdx.x >> 4);
      const bool valid = k < n;
      const RPatch* P = (const RPatch*)(items + (size_t)(valid ? k : 0) * sizeof(RPatch));
      const uint32_t depth = P->depth;
      const int dir = (int)((P->dirs >> depth) & 1u);
      float4 L, R;
      int my;
      split_cp(P, dir, lane, L, R, my);
      int slot = -1;
      if (lane == 0 && valid) slot = ctx.template reserve<BOUND>(2);
      slot = __shfl_sync(0xffffffffu, slot, 0, 16);
      if (valid && slot >= 0) {
        RPatch* l = (RPatch*)ctx.template out_ptr<BOUND>(slot);
        RPatch* r = (RPatch*)ctx.template out_ptr<BOUND>(slot + 1);
        cp_put(l, my, L);
        cp_put(r, my, R);
        if (lane == 0) split_headers(l, r, P->id, P->path, P->dirs, depth, dir);
      }
    }
  }

  static constexpr bool local_recursion(int lo, int hi) { return lo == BOUND && hi >= SPLIT; }
  // out buffers of a local-recursion kernel: none for Bound / Split / Dice (split nodes stay
  // in the warp, Dice items are published by the warps); a megakernel's Dice batches still
  // hand their grids to Shade through the out buffer
  static constexpr int local_out_cap(int, int hi, int t) { return (t == SHADE && hi >= DICE) ? 8 : 0; }

  // -------------------------------------------------------------- [Bound, Split] DFS
  // The [Bound, Split] group's own kernel (hi == Split): each warp works
  // claimed patches' split trees depth first, two nodes at a time (one per 16-thread group,
  // lane = control point, the node in registers): Bound, then either stage a Dice item,
  // cull, or split with de Casteljau over shuffles, keep the left child in registers and
  // push the right one on the warp's shared-memory stack.  A group without a node pops the
  // warp's stack (so both groups stay busy while either tree has pending children) and
  // only then claims the next item of the batch.  No block barrier: the warp's Dice items
  // are staged in shared memory and published by the warp itself (Ctx::publish_warp), and
  // the kernel is a sink group (no publisher warp), so warps go on to the next batch as
  // they finish.
  static constexpr int kDfsStack = 16;  // pending right children per warp: <= 2 root paths of <= 8
  static constexpr int kDfsStage = 8;   // Dice items a warp stages before publishing them
  struct DfsScratch {
    RPatch stack[kWarpsW][kDfsStack];
    RPatch stage[kWarpsW][kDfsStage];
    float4 M[2 * kWarpsW][4];            // each group's current frame matrix (rows)
  };
  static constexpr bool direct_publish(int lo, int hi, bool rtc) { return !rtc && lo == BOUND && hi == SPLIT; }
  static constexpr int direct_out_cap(int, int, int t) { return t == DICE ? kWarpsW * kDfsStage : 0; }

  template <int SS, class Ctx>
  static __device__ void exec_dfs(Ctx& ctx, const uint8_t* items, int n) {
    const Params& p = ctx.params();
    DfsScratch& ds = *(DfsScratch*)ctx.scratch();
    const int lane = threadIdx.x & 15, hw = threadIdx.x >> 4, half = hw & 1, warp = threadIdx.x >> 5;
    const unsigned hmask = 0xFFFFu << (16 * half);
    int* next = ctx.work_counter();
    RPatch* const stk = ds.stack[warp];
    RPatch* const stage = ds.stage[warp];
    int wsp = 0, wcnt = 0, nb = 0, nsp = 0;  // wsp, wcnt: warp-uniform
    bool have = false, first = false, presplit = false, drained = false;
    uint32_t mtag = 0;  // frame + 1 of the rows in ds.M[hw] (0: none), the same in every lane of the group
    float4 q = make_float4(0.f, 0.f, 0.f, 0.f);
    uint32_t id = 0, path = 0, dirs = 0, depth = 0;
    for (;;) {
      // groups without a node: the warp's pending children first, then the batch (one
      // claim atomic per warp); every decision here is warp-uniform
      const unsigned idle = __ballot_sync(0xffffffffu, !have && lane == 0);  // bit 0 / bit 16
      if (idle) {
        __syncwarp();  // last step's pushes come before these pops
        const int nidle = __popc(idle), rank = (half && (idle & 1u)) ? 1 : 0;
        const int from_stack = min(nidle, wsp);
        const int nclaim = drained ? 0 : nidle - from_stack;
        int kb = 0;
        if (nclaim > 0) {
          if ((threadIdx.x & 31) == 0) kb = atomicAdd(next, nclaim);
          kb = __shfl_sync(0xffffffffu, kb, 0);
        }
        if (!have) {
          const RPatch* src = nullptr;
          bool claimed = false;
          if (rank < from_stack) {
            src = &stk[wsp - 1 - rank];
          } else if (nclaim > 0 && kb + rank - from_stack < n) {
            src = (const RPatch*)(items + (size_t)(kb + rank - from_stack) * sizeof(RPatch));
            claimed = true;
          }
          if (src) {
            q = cp_get(src, lane);
            id = src->id;
            path = src->path;
            dirs = src->dirs;
            depth = src->depth;
            have = true;
            first = claimed;
            presplit = claimed && SS == SPLIT;  // a claimed Split item: its Bound already chose the direction
          }
        }
        if (nclaim > 0 && kb + nclaim >= n) drained = true;
        wsp -= from_stack;
        __syncwarp();  // the pops' reads come before this step's pushes
      }
      if (!__any_sync(0xffffffffu, have)) break;
      const uint32_t frame = frame_of(p, id);
      const bool reload = have && mtag != frame + 1;
      if (__any_sync(0xffffffffu, reload)) {
        __syncwarp();  // every read of the old rows is done
        if (reload) {
          ((float*)ds.M[hw])[lane] = __ldg(p.M + 16 * (size_t)frame + lane);
          mtag = frame + 1;
        }
        __syncwarp();
      }
      int dir = 0;
      int cls = bound_warp(p, q, depth, lane, have && !presplit, dir, ds.M[hw]);
      if (presplit) {
        cls = 1;
        dir = (int)((dirs >> depth) & 1u);
      }
      const unsigned long long node = ((unsigned long long)id << 12) | ((unsigned long long)(depth & 15u) << 8) | (path & 0xFFu);
      if (have && !presplit && !first) {  // a Bound task that never went through a ring
        ++nb;
        if (ctx.tracing() && lane == 0) ctx.template trace_local_id<BOUND>(node);
      }
      // Dice: stage the leaf in the warp's buffer (both groups may add one this step)
      const bool leaf = have && cls == 2;
      const unsigned lb = __ballot_sync(0xffffffffu, leaf && lane == 0);
      if (leaf) {
        RPatch* out = &stage[wcnt + ((half && (lb & 1u)) ? 1 : 0)];
        cp_put(out, lane, q);
        if (lane == 0) {
          out->id = id;
          out->path = path;
          out->dirs = dirs;
          out->depth = depth;
        }
      }
      wcnt += __popc(lb);
      const bool split = have && cls == 1;
      const unsigned sb = __ballot_sync(0xffffffffu, split && lane == 0);
      if (sb) {  // warp-uniform: the shuffles below run converged
        // de Casteljau at 1/2 (reading R-R6) of the curve through this lane's control point
        // along the split direction; same operations as split_cp, points from shuffles
        // Lane t of a curve (points a b c d) computes the de Casteljau levels at its own
        // position, h1 = (p_t + p_t+1) / 2, h2 = (h1_t + h1_t+1) / 2, h3 likewise, from the
        // next lane's value (lanes past the curve's end compute values nobody uses): h1 at
        // t = 0, 1, 2 is ab, bc, cd; h2 at t = 0, 1 is abc, bcd; h3 at t = 0 is m -- the same
        // operations in the same order as split_cp.  Right child point t is level 3 - t of
        // lane t itself, left child point t is level t of the curve's first lane.
        const int base = dir == 0 ? (lane & 3) : (lane & ~3), step = dir == 0 ? 4 : 1;
        const int t = dir == 0 ? (lane >> 2) : (lane & 3);
        float4 L, R;
#define VP_CASTELJAU(comp)                                                          \
  {                                                                                 \
    const float v = q.comp;                                                         \
    const float h1 = (v + __shfl_down_sync(0xffffffffu, v, step, 16)) * 0.5f;       \
    const float h2 = (h1 + __shfl_down_sync(0xffffffffu, h1, step, 16)) * 0.5f;     \
    const float h3 = (h2 + __shfl_down_sync(0xffffffffu, h2, step, 16)) * 0.5f;     \
    const float g1 = __shfl_sync(0xffffffffu, h1, base, 16);                        \
    const float g2 = __shfl_sync(0xffffffffu, h2, base, 16);                        \
    const float g3 = __shfl_sync(0xffffffffu, h3, base, 16);                        \
    L.comp = t == 0 ? v : t == 1 ? g1 : t == 2 ? g2 : g3;                           \
    R.comp = t == 0 ? h3 : t == 1 ? h2 : t == 2 ? h1 : v;                           \
  }
        VP_CASTELJAU(x) VP_CASTELJAU(y) VP_CASTELJAU(z)  // w stays 1 (R-S10)
#undef VP_CASTELJAU
        L.w = R.w = 1.0f;
        if (split) {
          const int slot = wsp + ((half && (sb & 1u)) ? 1 : 0);
          if (slot >= kDfsStack) {  // deeper than max_depth allows (cannot happen for valid seeds)
            ctx.abort(ABORT_GUARD);
            have = false;
          } else {
            if (!(first && presplit)) {  // a claimed Split item was counted when it was claimed
              ++nsp;
              if (ctx.tracing() && lane == 0) ctx.template trace_local_id<SPLIT>(node);
            }
            const uint32_t ndirs = (dirs & ~(1u << depth)) | ((uint32_t)dir << depth);
            RPatch* r = &stk[slot];
            cp_put(r, lane, R);
            if (lane == 0) {
              r->id = id;
              r->path = path | (1u << depth);
              r->dirs = ndirs;
              r->depth = depth + 1;
            }
            q = L;
            path &= ~(1u << depth);
            dirs = ndirs;
            depth += 1;
            first = presplit = false;
          }
        }
        wsp = min(wsp + __popc(sb), kDfsStack);
      }
      if (have && !split) have = false;  // diced or culled: the next node comes from the stack or the batch
      if (wcnt > kDfsStage - 2) {  // warp-uniform
        __syncwarp();
        ctx.template publish_warp<DICE>((const uint8_t*)stage, wcnt);
        wcnt = 0;
      }
    }
    if (wcnt > 0) {
      __syncwarp();
      ctx.template publish_warp<DICE>((const uint8_t*)stage, wcnt);
    }
    if (lane == 0) {
      ctx.template note_local_count_atomic<BOUND>(nb);
      ctx.template note_local_count_atomic<SPLIT>(nsp);
    }
  }

  // Block-local recursion (the paper fuses Bound into Split, L55): a kernel that runs Bound
  // and Split -- the [Bound, Split] group's own kernel or a megakernel -- works their
  // batches depth first (exec_dfs); a megakernel's later stages run as usual.
  template <int SS, int LO, int HI, class Ctx>
  static __device__ void exec_local(Ctx& ctx, const uint8_t* items, int n) {
    if constexpr (SS == DICE || SS == SHADE) exec<SS>(ctx, items, n);
    else exec_dfs<SS>(ctx, items, n);
  }

  // -------------------------------------------------------------- Dice (warp/patch)
  // One warp evaluates the 9x9 grid of patch P into `out` (readings R-R7, R-R9): the
  // separable Bernstein form, the 36 u-curve points C_a(v_j) staged as float4 in the (not
  // yet written) Q8-snap array s[] of `out`, then the 81 surface points (one lane per grid
  // row and 3 points), projection and Q8 snap.
  // Ms: the frame matrix rows in shared memory (fused chain), else read from p.M.
  // Bt (fused chain): the Bernstein weights B_b(j/8) as a [9][4] shared-memory table,
  // computed by bernstein() itself (bit-identical to evaluating it per point).
  // the u-curve point C_a(v_j), e = 9a + j, of patch P into the staging area (one lane)
  template <bool kSmemM>
  static __device__ __forceinline__ void dice_c(const RPatch* P, RGrid* out, int e, const float* Bt) {
    const int a = e / kNG, j = e - a * kNG;
    float Bv[4];
    if constexpr (kSmemM) {
      const float4 b4 = *(const float4*)&Bt[4 * j];
      Bv[0] = b4.x; Bv[1] = b4.y; Bv[2] = b4.z; Bv[3] = b4.w;
    } else {
      bernstein((float)j * 0.125f, Bv);
    }
    // P[a][0..3] of each coordinate plane: one 16-B load each
    const float4 X = *(const float4*)&P->x[4 * a], Y = *(const float4*)&P->y[4 * a], Z = *(const float4*)&P->z[4 * a];
    const float px[4] = {X.x, X.y, X.z, X.w}, py[4] = {Y.x, Y.y, Y.z, Y.w}, pz[4] = {Z.x, Z.y, Z.z, Z.w};
    float cx = 0.0f, cy = 0.0f, cz = 0.0f;
#pragma unroll
    for (int b = 0; b < 4; ++b) {
      cx = cx + Bv[b] * px[b];
      cy = cy + Bv[b] * py[b];
      cz = cz + Bv[b] * pz[b];
    }
    ((float4*)out->s)[e] = make_float4(cx, cy, cz, 0.0f);
  }

  // kHaveC: the caller already computed the u-curve points (the fused chain does both
  // patches of a pair in one loop: 72 points in 3 warp passes instead of 2 x 2).
  // Returns (warp-uniform) whether every grid point was snappable.
  template <bool kSmemM = false, bool kHaveC = false>
  static __device__ __forceinline__ bool dice_patch(const Params& p, const RPatch* P, RGrid* out, int lane,
                                                    const float4* Ms = nullptr, const float* Bt = nullptr) {
    const uint32_t frame = frame_of(p, P->id);
    const float* M = p.M + 16 * (size_t)frame;
    if constexpr (!kHaveC) {
      for (int e = lane; e < 4 * kNG; e += 32) dice_c<kSmemM>(P, out, e, Bt);  // C_a(v_j), e = 9a + j
      __syncwarp();
    }
    const float4* C = (const float4*)out->s;
    // Lanes 0..26: grid row j = lane / 3 (its u-curve points C_a(v_j) loaded once), points
    // i = i0 .. i0 + 2, i0 = 3 (lane % 3); g = 9j + i.  S(u_i, v_j) goes into o[g].xyz at once
    // (the staged C in s[] is still being read by other lanes, so s[] is written after the
    // next __syncwarp).
    const bool lw = lane < 3 * kNG;
    const int j = lane / 3, i0 = 3 * (lane - 3 * j), g0 = j * kNG + i0;
    if (lw) {
      float4 Cj[4];
#pragma unroll
      for (int a = 0; a < 4; ++a) Cj[a] = C[a * kNG + j];
#pragma unroll
      for (int r = 0; r < 3; ++r) {
        const int i = i0 + r;
        float Bu[4];
        if constexpr (kSmemM) {
          const float4 b4 = *(const float4*)&Bt[4 * i];
          Bu[0] = b4.x; Bu[1] = b4.y; Bu[2] = b4.z; Bu[3] = b4.w;
        } else {
          bernstein((float)i * 0.125f, Bu);
        }
        float x = 0.0f, y = 0.0f, z = 0.0f;
#pragma unroll
        for (int a = 0; a < 4; ++a) {
          x = x + Bu[a] * Cj[a].x;
          y = y + Bu[a] * Cj[a].y;
          z = z + Bu[a] * Cj[a].z;
        }
        out->o[g0 + r] = make_float4(x, y, z, 0.0f);
      }
    }
    __syncwarp();  // every C read before s[] is written
    bool ok_all = true;
    if (lw) {
#if VP_MS_REG
      float4 Mr[4];
      if constexpr (kSmemM) {
#pragma unroll
        for (int q = 0; q < 4; ++q) Mr[q] = Ms[q];
      }
#endif
#pragma unroll
      for (int r = 0; r < 3; ++r) {
        const int g = g0 + r;
        const float4 ov = out->o[g];  // this lane's own write
        const float x = ov.x, y = ov.y, z = ov.z;
        float4 c;
        if constexpr (kSmemM) {
          float cc[4];
#pragma unroll
          for (int q = 0; q < 4; ++q) {
#if VP_MS_REG
            const float4 m = Mr[q];
#else
            const float4 m = Ms[q];
#endif
            float acc = m.x * x;
            acc = acc + m.y * y;
            acc = acc + m.z * z;
            acc = acc + m.w;  // m.w * 1: exact, so the multiply is dropped
            cc[q] = acc;
          }
          c = make_float4(cc[0], cc[1], cc[2], cc[3]);
        } else {
          c = project(M, x, y, z, 1.0f);
        }
        float sx, sy, zs;
        screen(p, c, sx, sy, zs);
        // Shade only uses the Q8 fixed-point snap of (sx, sy): store it (reading R-R9)
        const float X = sx * 256.0f, Y = sy * 256.0f;
        const bool ok = fabsf(X) < 1073741824.0f && fabsf(Y) < 1073741824.0f;
        const int Xi = ok ? __float2int_rn(X) : INT_MIN, Yi = ok ? __float2int_rn(Y) : INT_MIN;
        out->o[g].w = zs;
        out->s[sidx(i0 + r, j)] = make_int2(Xi, Yi);
        ok_all = ok_all && ok;
      }
    }
    if (lane == 0) {
      out->id = P->id;
      out->path = P->path;
      out->depth = P->depth;
      out->dirs = P->dirs;
    }
    return __all_sync(0xffffffffu, ok_all);
  }

  template <class Ctx>
  static __device__ void dice(Ctx& ctx, const uint8_t* items, int n) {
    const Params& p = ctx.params();
    const int lane = threadIdx.x & 31;
    for (int r0 = 0; r0 < n; r0 += kThreads / 32) {
      const int k = r0 + (threadIdx.x >> 5);
      if (k >= n) break;  // warp-uniform
      int slot = 0;
      if (lane == 0) slot = ctx.template reserve<SHADE>();
      slot = __shfl_sync(0xffffffffu, slot, 0);
      if (slot < 0) continue;
      dice_patch(p, (const RPatch*)(items + (size_t)k * sizeof(RPatch)), (RGrid*)ctx.template out_ptr<SHADE>(slot), lane);
    }
  }

  // -------------------------------------------------------------- Shade (per micropolygon)
  // Micropolygon q = 8i + j of grid Gd: the quad (i,j)..(i+1,j+1), split into the
  // triangles (v0,v1,v2), (v0,v2,v3) (reading R-R8..R-R10).
  // kBoxed: the caller already established mp_box (valid frame, snappable corners, a pixel
  // centre in the box), so those early exits are skipped
  template <bool kBoxed = false>
  static __device__ __forceinline__ void shade_mp(const Params& p, const RGrid* Gd, int q) {
    const uint32_t frame = (Gd->id >> 12) - (uint32_t)p.frame_base, patch = Gd->id & 0xFFFu;
    if (!kBoxed && frame >= (uint32_t)p.n_frames) return;
    const int i = q >> 3, j = q & 7;
    const int g00 = j * kNG + i, g10 = j * kNG + i + 1, g01 = (j + 1) * kNG + i, g11 = (j + 1) * kNG + i + 1;
    // Coverage first: the two triangles cover exactly the pixel centres inside either
    // one, all within the quad's box; a micropolygon whose box holds no pixel centre
    // (most of them at config 5: ~0.25 px^2 each) writes nothing, so its shading is
    // never computed.
    const int si[4] = {sidx(i, j), sidx(i + 1, j), sidx(i + 1, j + 1), sidx(i, j + 1)};
    int vx[4], vy[4];
#pragma unroll
    for (int v = 0; v < 4; ++v) {
      const int2 sv = Gd->s[si[v]];
      vx[v] = sv.x;
      vy[v] = sv.y;
    }
    const int xmin = min(min(vx[0], vx[1]), min(vx[2], vx[3])), xmax = max(max(vx[0], vx[1]), max(vx[2], vx[3]));
    const int ymin = min(min(vy[0], vy[1]), min(vy[2], vy[3])), ymax = max(max(vy[0], vy[1]), max(vy[2], vy[3]));
    // an unsnappable corner is INT_MIN in both coordinates, hence the minimum
    if (!kBoxed && xmin == INT_MIN) return;
    // |coords| < 2^30: these int expressions cannot overflow
    int px0 = -((128 - xmin) >> 8), px1 = (xmax - 128) >> 8;  // ceil / floor of (v - 128) / 256
    int py0 = -((128 - ymin) >> 8), py1 = (ymax - 128) >> 8;
    px0 = max(px0, 0);
    py0 = max(py0, 0);
    px1 = min(px1, p.W - 1);
    py1 = min(py1, p.H - 1);
    if (!kBoxed && (px0 > px1 || py0 > py1)) return;
    const float4 o00 = Gd->o[g00], o10 = Gd->o[g10], o01 = Gd->o[g01], o11 = Gd->o[g11];
    const float e1[3] = {o10.x - o00.x, o10.y - o00.y, o10.z - o00.z};
    const float e2[3] = {o01.x - o00.x, o01.y - o00.y, o01.z - o00.z};
    float nx = e1[1] * e2[2] - e1[2] * e2[1];
    float ny = e1[2] * e2[0] - e1[0] * e2[2];
    float nz = e1[0] * e2[1] - e1[1] * e2[0];
    float nn = nx * nx + ny * ny;
    nn = nn + nz * nz;
    float s;
    if (nn == 0.0f) {
      s = 0.1f;
    } else {
      float d = nx * p.L[0] + ny * p.L[1];
      d = d + nz * p.L[2];
      float t = d / sqrtf(nn);
      if (!(t > 0.0f)) t = 0.0f;
      s = 0.1f + 0.9f * t;
    }
    const float zq = ((o00.w + o10.w) + (o11.w + o01.w)) * 0.25f;
    const uint32_t mp = (patch << 18) | ((Gd->path & 0xFFu) << 10) | ((Gd->depth & 0xFu) << 6) | (uint32_t)q;
    const unsigned long long key = ((unsigned long long)zkey(zq) << 32) | mp;
    FbRec* fb = (FbRec*)p.fb + (size_t)frame * p.W * p.H;
    if ((unsigned)xmax - (unsigned)xmin < (1u << 14) && (unsigned)ymax - (unsigned)ymin < (1u << 14)) {
      // int32 quad path: coordinates relative to the box corner, |products| < 2^29
      int ax[4], ay[4];
#pragma unroll
      for (int v = 0; v < 4; ++v) {
        ax[v] = vx[v] - xmin;
        ay[v] = vy[v] - ymin;
      }
      const int X0 = px0 * 256 + 128 - xmin, Y0 = py0 * 256 + 128 - ymin;
      TriEdges A, B;
      tri_setup(A, ax[0], ay[0], ax[1], ay[1], ax[2], ay[2], X0, Y0);
      tri_setup(B, ax[0], ay[0], ax[2], ay[2], ax[3], ay[3], X0, Y0);
      for (int py = py0; py <= py1; ++py) {
        int a0 = A.w[0], a1 = A.w[1], a2 = A.w[2], b0 = B.w[0], b1 = B.w[1], b2 = B.w[2];
        FbRec* row = fb + (size_t)py * p.W;
        for (int px = px0; px <= px1; ++px) {
          const bool in = (A.live && (a0 | a1 | a2) >= 0) || (B.live && (b0 | b1 | b2) >= 0);
          if (in) fb_min(row + px, key, s);  // idempotent: a pixel in both writes once
          a0 += A.dx[0]; a1 += A.dx[1]; a2 += A.dx[2];
          b0 += B.dx[0]; b1 += B.dx[1]; b2 += B.dx[2];
        }
#pragma unroll
        for (int k = 0; k < 3; ++k) {
          A.w[k] += A.dy[k];
          B.w[k] += B.dy[k];
        }
      }
    } else {
      raster_tri(p, fb, vx[0], vy[0], vx[1], vy[1], vx[2], vy[2], key, s);
      raster_tri(p, fb, vx[0], vy[0], vx[2], vy[2], vx[3], vy[3], key, s);
    }
  }

  template <class Ctx>
  static __device__ void shade(Ctx& ctx, const uint8_t* items, int n) {
    const Params& p = ctx.params();
    const int q = threadIdx.x & 63;
    for (int r0 = 0; r0 < n; r0 += kThreads / 64) {
      const int k = r0 + (threadIdx.x >> 6);
      if (k >= n) break;  // uniform per pair of warps
      shade_mp(p, (const RGrid*)(items + (size_t)k * sizeof(RGrid)), q);
    }
  }

  // -------------------------------------------------------------- RTC [Dice, Shade]
  // Warp-granular run-to-completion: each warp dices one patch into a
  // block-local grid slot and shades it itself, so the chain needs no block barrier
  // between the two stages.  The same arithmetic as dice_patch / shade_mp, restaged:
  // the frame matrix comes from shared memory, and only the micropolygons whose box
  // holds a pixel centre (~1 in 4 at config 5) are shaded, compacted onto the warp's lanes.
  static constexpr bool fused_rtc(int s, int hi) { return s == DICE && hi == SHADE; }

  // shade_mp's early exit alone: does micropolygon q's box hold a pixel centre?  (any grid)
  template <bool kFrame = true>
  static __device__ __forceinline__ bool mp_box(const Params& p, const RGrid* Gd, int q) {
    if (kFrame && (Gd->id >> 12) - (uint32_t)p.frame_base >= (uint32_t)p.n_frames) return false;
    const int i = q >> 3, j = q & 7;
    const int si[4] = {sidx(i, j), sidx(i + 1, j), sidx(i + 1, j + 1), sidx(i, j + 1)};
    int vx[4], vy[4];
#pragma unroll
    for (int v = 0; v < 4; ++v) {
      const int2 sv = Gd->s[si[v]];
      vx[v] = sv.x;
      vy[v] = sv.y;
    }
    const int xmin = min(min(vx[0], vx[1]), min(vx[2], vx[3])), xmax = max(max(vx[0], vx[1]), max(vx[2], vx[3]));
    const int ymin = min(min(vy[0], vy[1]), min(vy[2], vy[3])), ymax = max(max(vy[0], vy[1]), max(vy[2], vy[3]));
    // shade_mp's test max(c, 0) <= min(f, W - 1), c = ceil((xmin - 128) / 256), f = floor((xmax
    // - 128) / 256), restated without the divisions: c <= f <=> 256 f + 128 >= xmin, c <= W - 1
    // <=> xmin <= 256 (W - 1) + 128, 0 <= f <=> xmax >= 128 (same for y).  An unsnappable
    // corner is INT_MIN in both coordinates, so it is the minimum: xmin != INT_MIN.
    const bool inx = xmin != INT_MIN && xmax >= 128 && xmin <= p.W * 256 - 128 && ((xmax - 128) & ~255) + 128 >= xmin;
    const bool iny = ymax >= 128 && ymin <= p.H * 256 - 128 && ((ymax - 128) & ~255) + 128 >= ymin;
    return inx && iny;
  }
  template <int S0, int HI, class Ctx>
  static __device__ void exec_rtc_chain(Ctx& ctx, const uint8_t* items, int n) {
    static_assert(S0 == DICE && HI == SHADE, "only the [Dice, Shade] chain is fused");
    static_assert(Ctx::template cap<SHADE>() >= kWarpsW, "one grid slot per worker warp");
    const Params& p = ctx.params();
    const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
    ChainScratch& cs = *(ChainScratch*)ctx.scratch();
    uint8_t* list = cs.list[warp];
    // Patches are handed out dynamically: shade work per patch varies with its size on
    // screen, so a static warp -> patch map leaves warps idle at the round barrier.
    int* next = ctx.work_counter();
    if (threadIdx.x == 0) ctx.template note_local_count<SHADE>(n);  // Dice emits one grid per patch
    float* Bt = cs.B[warp];
    for (int e = lane; e < 36; e += 32) {
      float B4[4];
      bernstein((float)(e >> 2) * 0.125f, B4);
      Bt[e] = B4[e & 3];
    }
    // Two grids per warp: its grid slot in both out buffers (no other warp uses slot
    // `warp`, and the publisher never reads Shade slots of a fused chain).  Patches are
    // diced in pairs and the pixel-covering micropolygons of both are shaded in one pass:
    // at config 5 about a quarter of a grid's 64 micropolygons cover a pixel centre, so one
    // grid alone fills only half of the warp's shading lanes.
    RGrid* const g0 = (RGrid*)ctx.template out_ptr_in<SHADE>(0, warp);
    RGrid* const g1 = (RGrid*)ctx.template out_ptr_in<SHADE>(1, warp);
    for (;;) {
      int k = 0;
      if (lane == 0) k = atomicAdd(next, 2);
      k = __shfl_sync(0xffffffffu, k, 0);
      if (k >= n) break;
      const int np = min(2, n - k);
      const RPatch* P0 = (const RPatch*)(items + (size_t)k * sizeof(RPatch));
      const RPatch* P1 = P0 + (np > 1 ? 1 : 0);
      // both frame matrices (lanes 0..15: patch 0, 16..31: patch 1) and the u-curve points
      // of both patches (72 points, 3 passes)
      if ((lane >> 4) < np) {
        const RPatch* P = (lane >> 4) ? P1 : P0;
        ((float*)cs.M[warp][lane >> 4])[lane & 15] = __ldg(p.M + 16 * (size_t)frame_of(p, P->id) + (lane & 15));
      }
      for (int e2 = lane; e2 < 36 * np; e2 += 32) {
        const bool second = e2 >= 36;
        dice_c<true>(second ? P1 : P0, second ? g1 : g0, e2 - (second ? 36 : 0), Bt);
      }
      __syncwarp();
      int tot = 0;
#pragma unroll
      for (int j = 0; j < 2; ++j) {
        if (j >= np) break;
        RGrid* g = j ? g1 : g0;
        const RPatch* P = j ? P1 : P0;
        dice_patch<true, true>(p, P, g, lane, cs.M[warp][j], Bt);
        __syncwarp();
        if (lane == 0) ctx.template trace_local<SHADE>((const uint8_t*)g);
        const bool fv = (P->id >> 12) - (uint32_t)p.frame_base < (uint32_t)p.n_frames;  // per patch
        const bool a0 = fv && mp_box<false>(p, g, lane), a1 = fv && mp_box<false>(p, g, lane + 32);
        const unsigned m0 = __ballot_sync(0xffffffffu, a0), m1 = __ballot_sync(0xffffffffu, a1);
        const unsigned lt = (1u << lane) - 1u;
        const int c0 = __popc(m0);
        if (a0) list[tot + __popc(m0 & lt)] = (uint8_t)(lane | (j << 6));
        if (a1) list[tot + c0 + __popc(m1 & lt)] = (uint8_t)((lane + 32) | (j << 6));
        tot += c0 + __popc(m1);
      }
      __syncwarp();
      if (lane == 0) ctx.template note_units<SHADE>(tot);
      for (int t = lane; t < tot; t += 32) {
        const int e = list[t];
        shade_mp<true>(p, (e >> 6) ? g1 : g0, e & 63);
      }
      __syncwarp();  // the slots, the matrix and the list are rewritten next
    }
  }

  // -------------------------------------------------------------- sinks
  static cudaError_t init_run(const Params& p, cudaStream_t st);
  static cudaError_t finalize(const Params& p, cudaStream_t st);
  static bool output(const Params& p, int idx, void** ptr, size_t* bytes) {
    size_t npix = (size_t)p.n_frames * p.W * p.H;
    if (idx == 0) { *ptr = p.fb; *bytes = npix * sizeof(FbRec); return true; }
    if (idx == 1) { *ptr = p.colour; *bytes = npix * 16; return true; }
    return false;
  }
  static const char* validate(const Params& p) {
    if (p.W <= 0 || p.H <= 0 || p.W > 32767 || p.H > 32767) return "vp_reyes_params: bad W/H (int16 pixel ranges)";
    if (p.n_frames <= 0 || p.n_frames > (1 << 20)) return "vp_reyes_params: bad n_frames";
    if (p.patches_per_frame <= 0 || p.patches_per_frame > 4096) return "vp_reyes_params: patches_per_frame must be in [1, 4096]";
    if (p.max_depth < 0 || p.max_depth > 8) return "vp_reyes_params: max_depth must be in [0, 8] (8-bit path)";
    if (!p.M || !p.albedo || !p.fb || !p.colour) return "vp_reyes_params: M, albedo, fb, colour are required device pointers";
    if (((uintptr_t)p.fb & 15) || ((uintptr_t)p.colour & 15)) return "vp_reyes_params: fb and colour must be 16-B aligned";
    return nullptr;
  }
};

__global__ void k_reyes_clear(FbRec* fb, size_t n) {
  for (size_t i = blockIdx.x * (size_t)blockDim.x + threadIdx.x; i < n; i += (size_t)gridDim.x * blockDim.x) {
    FbRec r;
    r.key = ~0ull;
    r.s = 0.0f;
    r.pad = 0;
    fb[i] = r;
  }
}
// Resolve (sink): colour = albedo[patch of the winning micropolygon] * s (reading R-R11).
__global__ void k_reyes_resolve(const FbRec* __restrict__ fb, float4* __restrict__ colour, const float* __restrict__ albedo,
                                size_t n) {
  for (size_t i = blockIdx.x * (size_t)blockDim.x + threadIdx.x; i < n; i += (size_t)gridDim.x * blockDim.x) {
    FbRec r = fb[i];
    float4 c = make_float4(0.f, 0.f, 0.f, 0.f);
    if (r.key != ~0ull) {
      uint32_t patch = (uint32_t)(r.key >> 18) & 0xFFFu;
      const float* a = albedo + 4 * (size_t)patch;
      c = make_float4(a[0] * r.s, a[1] * r.s, a[2] * r.s, 1.0f);
    }
    colour[i] = c;
  }
}

cudaError_t ReyesF::init_run(const Params& p, cudaStream_t st) {
  size_t n = (size_t)p.n_frames * p.W * p.H;
  k_reyes_clear<<<(int)std::min<size_t>((n + 255) / 256, 148 * 16), 256, 0, st>>>((FbRec*)p.fb, n);
  return cudaGetLastError();
}
cudaError_t ReyesF::finalize(const Params& p, cudaStream_t st) {
  size_t n = (size_t)p.n_frames * p.W * p.H;
  k_reyes_resolve<<<(int)std::min<size_t>((n + 255) / 256, 148 * 16), 256, 0, st>>>((const FbRec*)p.fb, (float4*)p.colour, p.albedo, n);
  return cudaGetLastError();
}

const FamilyOps* family_reyes() {
  static FamilyImpl<ReyesF> f("reyes");
  return &f;
}

}  // namespace vp

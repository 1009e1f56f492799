// fam_raster.cu — triangle rasterization as VersaPipe stages (Fig. 16:
// Clip -> Interpolate -> Shade; Table 2: 4-B items).  Readings R-S1..R-S8 of DESIGN.md
// §2: the paper's Clip is Vertex + Clip here, Interpolate is Raster
// (triangle -> 8x8 tiles), Shade is Fragment (per-pixel coverage, depth, z-buffer
// atomicMin) plus a data-parallel colour resolve sink.  Compiled with -fmad=false:
// bit-identical to the CPU oracle.
//
// Items are triangle ids (4 B) and {tri, tile} pairs (8 B); per-triangle data lives in a
// 128-B global setup record (clip coordinates, then the fixed-point screen setup).
#include <limits.h>
#include <math.h>

#include <algorithm>

#include "../../include/vp.h"
#include "vp_family.cuh"

#ifndef VP_RASTER_MINB
#define VP_RASTER_MINB 3
#endif

namespace vp {

struct __align__(16) RSetup {   // 128 B per triangle
  float4 clip[3];               // Vertex -> Clip
  int X[3], Y[3];               // Q4 screen position (orientation-normalised order)
  float z[3];                   // z / w
  int px0, px1, py0, py1;       // pixel-centre range inside the bbox, clamped to the screen
  long long area;               // twice the signed area (> 0)
  int vi;                       // original vertex index of slot k in bits 2k..2k+1
  int pad[3];
};
static_assert(sizeof(RSetup) == 128, "setup record");

struct FragItem {
  uint32_t tri, tile;  // tile = ty << 16 | tx
};

__device__ __forceinline__ uint32_t rz_key(float z) {
  uint32_t b = __float_as_uint(z);
  return (b & 0x80000000u) ? ~b : (b | 0x80000000u);
}
template <class I>
__device__ __forceinline__ I r_edge(I ax, I ay, I bx, I by, I px, I py) {
  return (bx - ax) * (py - ay) - (by - ay) * (px - ax);
}
template <class I>
__device__ __forceinline__ bool r_owns(I ax, I ay, I bx, I by) {
  I dx = bx - ax, dy = by - ay;
  return dy > 0 || (dy == 0 && dx < 0);
}

// Coverage + barycentric weights at pixel (px, py) (R-S5/R-S6).  Exact integer edge
// functions (int32 when the triangle's box is < 2^14 Q4 units, else int64).
__device__ __forceinline__ bool frag_weights(const RSetup& s, int px, int py, float l[3]) {
  long long Px = (long long)px * 16 + 8, Py = (long long)py * 16 + 8;
  long long E0, E1, E2;
  bool i0, i1, i2;
  int xmin = min(s.X[0], min(s.X[1], s.X[2])), xmax = max(s.X[0], max(s.X[1], s.X[2]));
  int ymin = min(s.Y[0], min(s.Y[1], s.Y[2])), ymax = max(s.Y[0], max(s.Y[1], s.Y[2]));
  if (xmax - xmin < (1 << 14) && ymax - ymin < (1 << 14) && Px - xmin < (1 << 14) && Py - ymin < (1 << 14) &&
      Px - xmin >= -(1 << 14) && Py - ymin >= -(1 << 14)) {
    int ax = s.X[0] - xmin, ay = s.Y[0] - ymin, bx = s.X[1] - xmin, by = s.Y[1] - ymin, cx = s.X[2] - xmin,
        cy = s.Y[2] - ymin, qx = (int)(Px - xmin), qy = (int)(Py - ymin);
    int e0 = r_edge(bx, by, cx, cy, qx, qy), e1 = r_edge(cx, cy, ax, ay, qx, qy), e2 = r_edge(ax, ay, bx, by, qx, qy);
    i2 = e2 > 0 || (e2 == 0 && r_owns(ax, ay, bx, by));
    i0 = e0 > 0 || (e0 == 0 && r_owns(bx, by, cx, cy));
    i1 = e1 > 0 || (e1 == 0 && r_owns(cx, cy, ax, ay));
    E0 = e0;
    E1 = e1;
    E2 = e2;
  } else {
    long long ax = s.X[0], ay = s.Y[0], bx = s.X[1], by = s.Y[1], cx = s.X[2], cy = s.Y[2];
    E0 = r_edge(bx, by, cx, cy, Px, Py);
    E1 = r_edge(cx, cy, ax, ay, Px, Py);
    E2 = r_edge(ax, ay, bx, by, Px, Py);
    i2 = E2 > 0 || (E2 == 0 && r_owns(ax, ay, bx, by));
    i0 = E0 > 0 || (E0 == 0 && r_owns(bx, by, cx, cy));
    i1 = E1 > 0 || (E1 == 0 && r_owns(cx, cy, ax, ay));
  }
  if (!(i0 && i1 && i2)) return false;
  const float A = __ll2float_rn(s.area);
  l[0] = __ll2float_rn(E0) / A;
  l[1] = __ll2float_rn(E1) / A;
  l[2] = __ll2float_rn(E2) / A;
  return true;
}

struct RasterF {
  static constexpr int S = 4;
  static __host__ __device__ __forceinline__ unsigned long long n_setups(const vp_raster_params& p) {
    return (unsigned long long)p.n_tris << (p.near_clip ? 1 : 0);
  }
  static constexpr int VERTEX = 0, CLIP = 1, RASTER = 2, FRAGMENT = 3;
  static constexpr int kMaxTiles = 128;  // declared fan-out of Raster (10 x 10 for the generator's triangles)
  static constexpr int kinds[S] = {VP_RASTER_VERTEX, VP_RASTER_CLIP, VP_RASTER_RASTER, VP_RASTER_FRAGMENT};
  using Params = vp_raster_params;
  static constexpr int stride(int s) { return s == FRAGMENT ? 8 : 4; }
  static constexpr int threads_per_item(int s) { return s == RASTER ? 32 : s == FRAGMENT ? 64 : 1; }
  // (Vertex / Clip batches of 1024 were tried in round 2: no change for Vertex, Clip 20 ->
  // 18% of HBM under KBK, and the megakernel 3.2 -> 4.3 ms; a KBK wave of these stages is
  // a ~0.1 ms kernel of 2-10 rounds per block, so its ramp-up and tail bound it)
  static constexpr int max_batch(int s) { return s <= CLIP ? 256 : s == RASTER ? 32 : 32; }
  static constexpr int default_batch(int s) { return max_batch(s); }
  static constexpr int fanout(int s, int t) {
    return (t == s + 1) ? (s == RASTER ? kMaxTiles : s == CLIP ? 2 : 1) : 0;  // Clip: 0..2 (near clip)
  }
  // RTC groups must not expand Raster's fan-out block-locally from more than one claimed
  // batch: Raster may only be the first stage of an RTC group.
  static constexpr bool rtc_ok(int lo, int hi) { return !(lo < RASTER && hi >= RASTER); }
  // kernels running Raster: a 32-item Fragment staging area per warp for big triangles
  static constexpr int scratch_bytes(int lo, int hi) { return (lo <= RASTER && RASTER <= hi) ? kWarpsW * 32 * 8 : 0; }
  static constexpr int default_cap_log2(int s) { return s == FRAGMENT ? 22 : 21; }
  static constexpr int min_blocks(int, int, bool) { return VP_RASTER_MINB; }

  template <int s>
  static __device__ unsigned long long item_id(const uint8_t* it) {
    if constexpr (s == FRAGMENT) {
      const FragItem* f = (const FragItem*)it;
      return ((unsigned long long)f->tri << 32) | f->tile;
    } else {
      return *(const uint32_t*)it;
    }
  }

  template <int s, class Ctx>
  static __device__ void exec(Ctx& ctx, const uint8_t* items, int n) {
    if constexpr (s == VERTEX) vertex(ctx, items, n);
    else if constexpr (s == CLIP) clip(ctx, items, n);
    else if constexpr (s == RASTER) raster(ctx, items, n);
    else fragment(ctx, items, n);
  }

  // ------------------------------------------------------------ Vertex (1 thread/tri)
  template <class Ctx>
  static __device__ void vertex(Ctx& ctx, const uint8_t* items, int n) {
    const Params& p = ctx.params();
    RSetup* setup = (RSetup*)p.setup;
    for (int k = threadIdx.x; k < n; k += kThreads) {
      const uint32_t tri = ((const uint32_t*)items)[k];
      if (tri >= (uint32_t)p.n_tris) continue;
      const float4* v = (const float4*)p.pos + 3 * (size_t)tri;
#pragma unroll
      for (int q = 0; q < 3; ++q) {
        const float4 x = __ldg(v + q);
        float c[4];
#pragma unroll
        for (int r = 0; r < 4; ++r) {
          float acc = __ldg(p.M + 4 * r + 0) * x.x;
          acc = acc + __ldg(p.M + 4 * r + 1) * x.y;
          acc = acc + __ldg(p.M + 4 * r + 2) * x.z;
          acc = acc + __ldg(p.M + 4 * r + 3) * x.w;
          c[r] = acc;
        }
        setup[p.near_clip ? 2 * (size_t)tri : tri].clip[q] = make_float4(c[0], c[1], c[2], c[3]);
      }
      ctx.template emit<CLIP>(&tri);
    }
  }

  // Setup of one (sub-)triangle from its clip coordinates (R-S2..R-S4): trivial reject,
  // w cull, Q4 snap, orientation, pixel range.  Returns false if it is culled.
  static __device__ __forceinline__ bool setup_one(const Params& p, const float4 c[3], RSetup& s) {
    bool o0 = true, o1 = true, o2 = true, o3 = true, o4 = true, o5 = true;
#pragma unroll
    for (int q = 0; q < 3; ++q) {
      o0 &= c[q].x < -c[q].w;
      o1 &= c[q].x > c[q].w;
      o2 &= c[q].y < -c[q].w;
      o3 &= c[q].y > c[q].w;
      o4 &= c[q].z < 0.0f;
      o5 &= c[q].z > c[q].w;
    }
    if (o0 || o1 || o2 || o3 || o4 || o5) return false;  // trivial reject
    if (!(c[0].w > 1e-6f) || !(c[1].w > 1e-6f) || !(c[2].w > 1e-6f)) return false;
    long long X[3], Y[3];
    float Z[3];
    bool ok = true;
#pragma unroll
    for (int q = 0; q < 3; ++q) {
      const float w = c[q].w;
      const float sx = ((c[q].x / w) * 0.5f + 0.5f) * (float)p.W;
      const float sy = ((c[q].y / w) * 0.5f + 0.5f) * (float)p.H;
      const float fx = sx * 16.0f, fy = sy * 16.0f;
      if (!(fabsf(fx) < 1073741824.0f) || !(fabsf(fy) < 1073741824.0f)) ok = false;
      X[q] = __float2ll_rn(fx);
      Y[q] = __float2ll_rn(fy);
      Z[q] = c[q].z / w;
    }
    if (!ok) return false;
    long long area = r_edge(X[0], Y[0], X[1], Y[1], X[2], Y[2]);
    if (area == 0) return false;
    int o[3] = {0, 1, 2};
    if (area < 0) {
      o[1] = 2;
      o[2] = 1;
      area = -area;
    }
    long long xmin = min(X[0], min(X[1], X[2])), xmax = max(X[0], max(X[1], X[2]));
    long long ymin = min(Y[0], min(Y[1], Y[2])), ymax = max(Y[0], max(Y[1], Y[2]));
    long long px0 = -((-(xmin - 8)) >> 4), px1 = (xmax - 8) >> 4;  // ceil / floor of (v - 8) / 16
    long long py0 = -((-(ymin - 8)) >> 4), py1 = (ymax - 8) >> 4;
    px0 = max(px0, 0ll);
    py0 = max(py0, 0ll);
    px1 = min(px1, (long long)p.W - 1);
    py1 = min(py1, (long long)p.H - 1);
    if (px0 > px1 || py0 > py1) return false;
    int vi = 0;
#pragma unroll
    for (int q = 0; q < 3; ++q) {
      const int src = q == 0 ? o[0] : q == 1 ? o[1] : o[2];
      s.X[q] = (int)(src == 0 ? X[0] : src == 1 ? X[1] : X[2]);
      s.Y[q] = (int)(src == 0 ? Y[0] : src == 1 ? Y[1] : Y[2]);
      s.z[q] = src == 0 ? Z[0] : src == 1 ? Z[1] : Z[2];
      vi |= src << (2 * q);
    }
    s.px0 = (int)px0;
    s.px1 = (int)px1;
    s.py0 = (int)py0;
    s.py1 = (int)py1;
    s.area = area;
    s.vi = vi;
    return true;
  }

  // ------------------------------------------------------------ Clip (1 thread/tri)
  template <class Ctx>
  static __device__ void clip(Ctx& ctx, const uint8_t* items, int n) {
    const Params& p = ctx.params();
    RSetup* setup = (RSetup*)p.setup;
    for (int k = threadIdx.x; k < n; k += kThreads) {
      const uint32_t tri = ((const uint32_t*)items)[k];
      if (tri >= (uint32_t)p.n_tris) continue;
      if (!p.near_clip) {
        RSetup& s = setup[tri];
        const float4 c[3] = {s.clip[0], s.clip[1], s.clip[2]};
        if (setup_one(p, c, s)) ctx.template emit<RASTER>(&tri);
        continue;
      }
      // Near-plane clip (R-S9): Sutherland-Hodgman against z >= 0, fan into sub-triangles
      // 2 tri + j.  Clip coordinates were left in setup[2 tri] by Vertex.
      const float4 c[3] = {setup[2 * tri].clip[0], setup[2 * tri].clip[1], setup[2 * tri].clip[2]};
      {
        bool o0 = true, o1 = true, o2 = true, o3 = true, o4 = true, o5 = true;
#pragma unroll
        for (int q = 0; q < 3; ++q) {
          o0 &= c[q].x < -c[q].w;
          o1 &= c[q].x > c[q].w;
          o2 &= c[q].y < -c[q].w;
          o3 &= c[q].y > c[q].w;
          o4 &= c[q].z < 0.0f;
          o5 &= c[q].z > c[q].w;
        }
        if (o0 || o1 || o2 || o3 || o4 || o5) continue;
      }
      // The polygon is kept as up to 4 (source edge q, t) pairs -- t < 0: vertex q itself,
      // else the point a + t (b - a) on edge q (a = vertex q, b = vertex q+1) -- written by
      // select into fixed slots, so it stays in 8 registers (no local-memory array).
      int pe0 = 0, pe1 = 0, pe2 = 0, pe3 = 0;
      float pt0 = -1.f, pt1 = -1.f, pt2 = -1.f, pt3 = -1.f;
      int np = 0;
#pragma unroll
      for (int q = 0; q < 3; ++q) {
        const float4 a = c[q], b = c[(q + 1) % 3];
        const bool ina = a.z >= 0.0f, inb = b.z >= 0.0f;
        if (ina) {
          if (np == 0) pe0 = q, pt0 = -1.f;
          if (np == 1) pe1 = q, pt1 = -1.f;
          if (np == 2) pe2 = q, pt2 = -1.f;
          if (np == 3) pe3 = q, pt3 = -1.f;  // v0 in, v1 out, v2 in: v2 is the 4th vertex
          ++np;
        }
        if (ina != inb) {
          const float t = a.z / (a.z - b.z);
          if (np == 0) pe0 = q, pt0 = t;
          if (np == 1) pe1 = q, pt1 = t;
          if (np == 2) pe2 = q, pt2 = t;
          if (np == 3) pe3 = q, pt3 = t;
          ++np;
        }
      }
      const float4* col = (const float4*)p.col + 3 * (size_t)tri;
      float4* ccol = (float4*)p.ccol;
      // polygon vertex (q, t): clip coordinates and colour
      auto vert = [&](int q, float t, float4& v, float4& cv) {
        const float4 a = q == 0 ? c[0] : q == 1 ? c[1] : c[2];
        const int qb = q == 2 ? 0 : q + 1;
        const float4 ca = __ldg(col + q);
        if (t < 0.0f) {
          v = a;
          cv = ca;
        } else {
          const float4 b = qb == 0 ? c[0] : qb == 1 ? c[1] : c[2];
          const float4 cb = __ldg(col + qb);
          v = make_float4(a.x + t * (b.x - a.x), a.y + t * (b.y - a.y), 0.0f, a.w + t * (b.w - a.w));
          cv = make_float4(ca.x + t * (cb.x - ca.x), ca.y + t * (cb.y - ca.y), ca.z + t * (cb.z - ca.z),
                           ca.w + t * (cb.w - ca.w));
        }
      };
#pragma unroll
      for (int j = 0; j < 2; ++j) {
        if (j + 2 >= np) break;
        // fan triangle (p0, p(j+1), p(j+2))
        float4 v[3], cv[3];
        vert(pe0, pt0, v[0], cv[0]);
        vert(j == 0 ? pe1 : pe2, j == 0 ? pt1 : pt2, v[1], cv[1]);
        vert(j == 0 ? pe2 : pe3, j == 0 ? pt2 : pt3, v[2], cv[2]);
        const uint32_t sub = 2 * tri + (uint32_t)j;
        RSetup& s = setup[sub];
        if (!setup_one(p, v, s)) continue;
#pragma unroll
        for (int q = 0; q < 3; ++q) {
          const int src = (s.vi >> (2 * q)) & 3;
          ccol[3 * (size_t)sub + q] = src == 0 ? cv[0] : src == 1 ? cv[1] : cv[2];
        }
        ctx.template emit<RASTER>(&sub);
      }
    }
  }

  // ------------------------------------------------------------ Raster (warp/tri)
  template <class Ctx>
  static __device__ void raster(Ctx& ctx, const uint8_t* items, int n) {
    const Params& p = ctx.params();
    const RSetup* setup = (const RSetup*)p.setup;
    const int lane = threadIdx.x & 31;
    for (int r0 = 0; r0 < n; r0 += kWarpsW) {
      const int k = r0 + (threadIdx.x >> 5);
      if (k >= n) break;  // warp-uniform
      const uint32_t tri = ((const uint32_t*)items)[k];  // sub-triangle id in near-clip mode
      if ((unsigned long long)tri >= n_setups(p)) continue;
      const RSetup& s = setup[tri];
      const int tx0 = s.px0 >> 3, tx1 = s.px1 >> 3, ty0 = s.py0 >> 3, ty1 = s.py1 >> 3;
      const int ntx = tx1 - tx0 + 1, nt = ntx * (ty1 - ty0 + 1);
      const long long X[3] = {s.X[0], s.X[1], s.X[2]}, Y[3] = {s.Y[0], s.Y[1], s.Y[2]};
      // A triangle with more candidate tiles than the declared fan-out (a big or near-camera
      // triangle; reading R-S8) does not go through the block's out buffer: the warp
      // publishes its tiles to the Fragment ring itself, 32 at a time (same items, same
      // order-free result; the ring must hold one wave's big triangles in KBK mode).
      const bool big = nt > kMaxTiles;  // warp-uniform
      FragItem* const stage = (FragItem*)ctx.scratch() + 32 * (threadIdx.x >> 5);
      for (int b = 0; b < nt; b += 32) {
        const int t = b + lane;
        bool emit = false;
        int tx = 0, ty = 0;
        if (t < nt) {
          ty = ty0 + t / ntx;
          tx = tx0 + t % ntx;
          long long x0 = max((long long)tx * 8, (long long)s.px0), x1 = min((long long)tx * 8 + 7, (long long)s.px1);
          long long y0 = max((long long)ty * 8, (long long)s.py0), y1 = min((long long)ty * 8 + 7, (long long)s.py1);
          const long long cx[2] = {x0 * 16 + 8, x1 * 16 + 8}, cy[2] = {y0 * 16 + 8, y1 * 16 + 8};
          bool rejected = false;
#pragma unroll
          for (int e = 0; e < 3; ++e) {
            const int a = e, c = (e + 1) % 3;
            bool all_out = true;
#pragma unroll
            for (int i = 0; i < 2; ++i)
#pragma unroll
              for (int j = 0; j < 2; ++j)
                if (r_edge(X[a], Y[a], X[c], Y[c], cx[i], cy[j]) >= 0) all_out = false;
            rejected |= all_out;
          }
          emit = !rejected;
        }
        const unsigned m = __ballot_sync(0xffffffffu, emit);
        if (big) {
          if (emit) {
            FragItem* out = &stage[__popc(m & ((1u << lane) - 1u))];
            out->tri = tri;
            out->tile = ((uint32_t)ty << 16) | (uint32_t)tx;
          }
          if (m) {
            __syncwarp();
            ctx.template publish_warp<FRAGMENT>((const uint8_t*)stage, __popc(m));
          }
          continue;
        }
        // warp-aggregated reservation of the surviving tiles (one smem atomic per warp)
        int base = 0;
        if (lane == 0 && m) base = ctx.template reserve<FRAGMENT>(__popc(m));
        base = __shfl_sync(0xffffffffu, base, 0);
        if (emit && base >= 0) {
          FragItem* out = (FragItem*)ctx.template out_ptr<FRAGMENT>(base + __popc(m & ((1u << lane) - 1u)));
          out->tri = tri;
          out->tile = ((uint32_t)ty << 16) | (uint32_t)tx;
        }
      }
    }
  }

  // ------------------------------------------------------------ Fragment (64 thr/tile)
  template <class Ctx>
  static __device__ void fragment(Ctx& ctx, const uint8_t* items, int n) {
    const Params& p = ctx.params();
    const RSetup* setup = (const RSetup*)p.setup;
    unsigned long long* fb = (unsigned long long*)p.fb;
    const int q = threadIdx.x & 63;
    for (int r0 = 0; r0 < n; r0 += kThreads / 64) {
      const int k = r0 + (threadIdx.x >> 6);
      if (k >= n) break;
      const FragItem f = ((const FragItem*)items)[k];
      if ((unsigned long long)f.tri >= n_setups(p)) continue;
      const RSetup& s = setup[f.tri];
      const int px = (int)(f.tile & 0xFFFFu) * 8 + (q & 7), py = (int)(f.tile >> 16) * 8 + (q >> 3);
      if (px < s.px0 || px > s.px1 || py < s.py0 || py > s.py1) continue;
      float l[3];
      if (!frag_weights(s, px, py, l)) continue;
      float z = l[0] * s.z[0] + l[1] * s.z[1];
      z = z + l[2] * s.z[2];
      if (!(z >= 0.0f && z <= 1.0f)) continue;
      const unsigned long long key = ((unsigned long long)rz_key(z) << 32) | f.tri;
      atomicMin(fb + (size_t)py * p.W + px, key);  // z-buffer: 64-bit RED.MIN at L2
    }
  }

  static cudaError_t init_run(const Params& p, cudaStream_t st);
  static cudaError_t finalize(const Params& p, cudaStream_t st);
  static bool output(const Params& p, int idx, void** ptr, size_t* bytes) {
    size_t npix = (size_t)p.W * p.H;
    if (idx == 0) { *ptr = p.fb; *bytes = npix * 8; return true; }
    if (idx == 1) { *ptr = p.colour; *bytes = npix * 16; return true; }
    return false;
  }
  static const char* validate(const Params& p) {
    if (p.W <= 0 || p.H <= 0 || p.W > 65535 || p.H > 65535) return "vp_raster_params: bad W/H";
    if (p.n_tris <= 0 || p.n_tris > (1ll << 31)) return "vp_raster_params: bad n_tris";
    if (!p.M || !p.pos || !p.col || !p.setup || !p.fb || !p.colour) return "vp_raster_params: M, pos, col, setup, fb, colour required";
    if (p.near_clip != 0 && p.near_clip != 1) return "vp_raster_params: near_clip must be 0 or 1";
    if (p.near_clip && (!p.ccol || ((uintptr_t)p.ccol & 15))) return "vp_raster_params: near_clip needs a 16-B aligned ccol";
    if (((uintptr_t)p.setup & 127) || ((uintptr_t)p.pos & 15) || ((uintptr_t)p.colour & 15))
      return "vp_raster_params: setup must be 128-B aligned; pos, colour 16-B aligned";
    return nullptr;
  }
};

__global__ void k_raster_clear(unsigned long long* fb, size_t n) {
  for (size_t i = blockIdx.x * (size_t)blockDim.x + threadIdx.x; i < n; i += (size_t)gridDim.x * blockDim.x) fb[i] = ~0ull;
}
// Resolve (sink, R-S7): colour of the winning triangle, re-derived at the pixel centre.
__global__ void k_raster_resolve(vp_raster_params p) {
  const size_t npix = (size_t)p.W * p.H;
  const RSetup* setup = (const RSetup*)p.setup;
  const unsigned long long* fb = (const unsigned long long*)p.fb;
  float4* colour = (float4*)p.colour;
  for (size_t i = blockIdx.x * (size_t)blockDim.x + threadIdx.x; i < npix; i += (size_t)gridDim.x * blockDim.x) {
    const unsigned long long key = fb[i];
    float4 c = make_float4(0.f, 0.f, 0.f, 0.f);
    if (key != ~0ull) {
      const uint32_t tri = (uint32_t)(key & 0xFFFFFFFFu);
      const RSetup& s = setup[tri];
      float l[3];
      if (frag_weights(s, (int)(i % p.W), (int)(i / p.W), l)) {
        float4 c0, c1, c2;
        if (p.near_clip) {  // sub-triangle colours, already in setup order
          const float4* cc = (const float4*)p.ccol + 3 * (size_t)tri;
          c0 = cc[0], c1 = cc[1], c2 = cc[2];
        } else {
          const float4* col = (const float4*)p.col + 3 * (size_t)tri;
          c0 = col[s.vi & 3], c1 = col[(s.vi >> 2) & 3], c2 = col[(s.vi >> 4) & 3];
        }
        float r = l[0] * c0.x + l[1] * c1.x;
        r = r + l[2] * c2.x;
        float g = l[0] * c0.y + l[1] * c1.y;
        g = g + l[2] * c2.y;
        float b = l[0] * c0.z + l[1] * c1.z;
        b = b + l[2] * c2.z;
        c = make_float4(r, g, b, 1.0f);
      } else {
        c = make_float4(-1.f, -1.f, -1.f, -1.f);  // cannot happen (winner covers its pixel)
      }
    }
    colour[i] = c;
  }
}

cudaError_t RasterF::init_run(const Params& p, cudaStream_t st) {
  size_t n = (size_t)p.W * p.H;
  k_raster_clear<<<(int)std::min<size_t>((n + 255) / 256, 148 * 8), 256, 0, st>>>((unsigned long long*)p.fb, n);
  return cudaGetLastError();
}
cudaError_t RasterF::finalize(const Params& p, cudaStream_t st) {
  size_t n = (size_t)p.W * p.H;
  k_raster_resolve<<<(int)std::min<size_t>((n + 255) / 256, 148 * 8), 256, 0, st>>>(p);
  return cudaGetLastError();
}

const FamilyOps* family_raster() {
  static FamilyImpl<RasterF> f("raster");
  return &f;
}

}  // namespace vp

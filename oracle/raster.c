/* raster.c — CPU ORACLE (test infrastructure only): triangle rasterization.
 *
 * PAPER.md L59 (Fig. 16: Clip -> Interpolate -> Shade; "100 cubes"), Table 1 L43 (3
 * stages, linear, dynamic), Table 2 L51 (4-B items).  The paper gives no formulas; the
 * arithmetic follows SURVEY §8(c-5) with the readings of DESIGN.md §2 (R-S1..R-S8):
 *
 *  Vertex(tri):   clip_k = M . p_k, row r = ((M[r0]x + M[r1]y) + M[r2]z) + M[r3]w.
 *  Clip(tri):     trivial reject if all 3 vertices are outside one of the planes
 *                 x<-w, x>w, y<-w, y>w, z<0, z>w; cull if any w <= 1e-6;
 *                 screen s = ((c/w)*0.5+0.5)*W, snapped to Q4: X = rint(s*16); z = z/w;
 *                 area2 = E(v0,v1,v2) in int64, 0 culls, < 0 swaps v1,v2 (orientation
 *                 normalised); pixel range = pixel centres inside the bbox, clamped to
 *                 the screen; empty culls.
 *  Raster(tri):   one {tri, tile} per 8x8 tile meeting the pixel range that no single
 *                 edge rejects: an edge rejects a tile when E < 0 at all four corner
 *                 sample points of the tile's part of the pixel range.
 *  Fragment:      per pixel centre (16px+8, 16py+8) of the tile in the pixel range:
 *                 inside iff every edge has E > 0 or (E == 0 and the edge owns it,
 *                 dy > 0 || (dy == 0 && dx < 0)); l0 = (float)E(v1,v2,P)/(float)area2,
 *                 l1 = E(v2,v0,P)/area2, l2 = E(v0,v1,P)/area2; z = (l0 z0 + l1 z1) + l2 z2;
 *                 discard unless 0 <= z <= 1; keep min key (zkey(z) << 32 | tri).
 *  Resolve:       colour = (l0 c0 + l1 c1) + l2 c2 of the winning triangle, alpha 1.
 *
 *  Near-plane clipping (sc->near_clip != 0, reading R-S9 of DESIGN.md
 *  §2): after the trivial reject, a triangle with a vertex at z < 0 is clipped against
 *  the plane z = 0 by Sutherland-Hodgman (edges v0v1, v1v2, v2v0 in order: keep a vertex
 *  with z >= 0; where an edge changes side, t = za / (za - zb) and every clip coordinate
 *  and colour channel is a + t (b - a), z set to exactly 0).  The 3- or 4-gon (p0..pn-1)
 *  fans into triangles (p0, p(j+1), p(j+2)), j = 0..n-3, each set up as above under the
 *  sub-triangle id 2 tri + j, which replaces tri in the depth key.  Clip's fan-out is 0..2.
 */
#include <math.h>
#include <stdlib.h>
#include <string.h>

#include "oracle.h"

typedef struct rsetup {
  int64_t X[3], Y[3];
  float z[3];
  int32_t vi[3]; /* vertex order after orientation normalisation */
  int64_t area;
  int32_t px0, px1, py0, py1;
  float c[3][4]; /* near-clip mode: vertex colours in setup order */
} rsetup;

static uint32_t r_zkey(float z) {
  uint32_t b;
  memcpy(&b, &z, 4);
  return (b & 0x80000000u) ? ~b : (b | 0x80000000u);
}

static int64_t r_edge(int64_t ax, int64_t ay, int64_t bx, int64_t by, int64_t px, int64_t py) {
  return (bx - ax) * (py - ay) - (by - ay) * (px - ax);
}
static int r_owns(int64_t ax, int64_t ay, int64_t bx, int64_t by) {
  int64_t dx = bx - ax, dy = by - ay;
  return dy > 0 || (dy == 0 && dx < 0);
}
static int64_t fdiv16(int64_t a) { return a >= 0 ? a / 16 : -((-a + 15) / 16); }

/* Vertex stage: clip-space positions of the 3 vertices. */
void orc_raster_vertex(const orc_raster_scene* sc, uint32_t tri, float clip[3][4]) {
  const float* p = sc->pos + 12 * (size_t)tri;
  for (int k = 0; k < 3; ++k) {
    const float* v = p + 4 * k;
    for (int r = 0; r < 4; ++r) {
      float acc = sc->M[4 * r + 0] * v[0];
      acc = acc + sc->M[4 * r + 1] * v[1];
      acc = acc + sc->M[4 * r + 2] * v[2];
      acc = acc + sc->M[4 * r + 3] * v[3];
      clip[k][r] = acc;
    }
  }
}

/* Clip stage: returns 1 and fills the setup if the triangle survives. */
static int clip_setup(const orc_raster_scene* sc, const float clip[3][4], rsetup* s) {
  /* trivial reject: all three outside one plane */
  int out[6] = {1, 1, 1, 1, 1, 1};
  for (int k = 0; k < 3; ++k) {
    float x = clip[k][0], y = clip[k][1], z = clip[k][2], w = clip[k][3];
    out[0] &= x < -w;
    out[1] &= x > w;
    out[2] &= y < -w;
    out[3] &= y > w;
    out[4] &= z < 0.0f;
    out[5] &= z > w;
  }
  for (int i = 0; i < 6; ++i)
    if (out[i]) return 0;
  for (int k = 0; k < 3; ++k)
    if (!(clip[k][3] > 1e-6f)) return 0;
  int64_t X[3], Y[3];
  float Z[3];
  for (int k = 0; k < 3; ++k) {
    float w = clip[k][3];
    float sx = ((clip[k][0] / w) * 0.5f + 0.5f) * (float)sc->W;
    float sy = ((clip[k][1] / w) * 0.5f + 0.5f) * (float)sc->H;
    float fx = sx * 16.0f, fy = sy * 16.0f;
    if (!(fabsf(fx) < 1073741824.0f) || !(fabsf(fy) < 1073741824.0f)) return 0;
    X[k] = (int64_t)rintf(fx);
    Y[k] = (int64_t)rintf(fy);
    Z[k] = clip[k][2] / w;
  }
  int64_t area = r_edge(X[0], Y[0], X[1], Y[1], X[2], Y[2]);
  if (area == 0) return 0;
  int o[3] = {0, 1, 2};
  if (area < 0) {
    o[1] = 2;
    o[2] = 1;
    area = -area;
  }
  for (int k = 0; k < 3; ++k) {
    s->X[k] = X[o[k]];
    s->Y[k] = Y[o[k]];
    s->z[k] = Z[o[k]];
    s->vi[k] = o[k];
  }
  s->area = area;
  int64_t xmin = X[0], xmax = X[0], ymin = Y[0], ymax = Y[0];
  for (int k = 1; k < 3; ++k) {
    if (X[k] < xmin) xmin = X[k];
    if (X[k] > xmax) xmax = X[k];
    if (Y[k] < ymin) ymin = Y[k];
    if (Y[k] > ymax) ymax = Y[k];
  }
  int64_t px0 = -fdiv16(-(xmin - 8)), px1 = fdiv16(xmax - 8);
  int64_t py0 = -fdiv16(-(ymin - 8)), py1 = fdiv16(ymax - 8);
  if (px0 < 0) px0 = 0;
  if (py0 < 0) py0 = 0;
  if (px1 > sc->W - 1) px1 = sc->W - 1;
  if (py1 > sc->H - 1) py1 = sc->H - 1;
  if (px0 > px1 || py0 > py1) return 0;
  s->px0 = (int32_t)px0;
  s->px1 = (int32_t)px1;
  s->py0 = (int32_t)py0;
  s->py1 = (int32_t)py1;
  return 1;
}

/* Near-plane clip (R-S9): polygon of the triangle clipped against z >= 0, fanned into
 * sub-triangles 2 tri + j.  Returns the number of surviving sub-triangles; alive[j] set. */
static int near_clip_setup(const orc_raster_scene* sc, uint32_t tri, const float clip[3][4], rsetup s[2],
                           int alive[2]) {
  alive[0] = alive[1] = 0;
  int out[6] = {1, 1, 1, 1, 1, 1};
  for (int k = 0; k < 3; ++k) {
    float x = clip[k][0], y = clip[k][1], z = clip[k][2], w = clip[k][3];
    out[0] &= x < -w;
    out[1] &= x > w;
    out[2] &= y < -w;
    out[3] &= y > w;
    out[4] &= z < 0.0f;
    out[5] &= z > w;
  }
  for (int i = 0; i < 6; ++i)
    if (out[i]) return 0;
  const float* col = sc->col + 12 * (size_t)tri;
  float P[4][4], C[4][4];
  int n = 0;
  for (int k = 0; k < 3; ++k) {
    const float* a = clip[k];
    const float* b = clip[(k + 1) % 3];
    const float* ca = col + 4 * k;
    const float* cb = col + 4 * ((k + 1) % 3);
    int ina = a[2] >= 0.0f, inb = b[2] >= 0.0f;
    if (ina) {
      memcpy(P[n], a, sizeof(float[4]));
      memcpy(C[n], ca, sizeof(float[4]));
      ++n;
    }
    if (ina != inb) {
      float t = a[2] / (a[2] - b[2]);
      for (int r = 0; r < 4; ++r) {
        P[n][r] = a[r] + t * (b[r] - a[r]);
        C[n][r] = ca[r] + t * (cb[r] - ca[r]);
      }
      P[n][2] = 0.0f;
      ++n;
    }
  }
  int m = 0;
  for (int j = 0; j + 2 < n; ++j) {
    int idx[3] = {0, j + 1, j + 2};
    float v[3][4];
    for (int k = 0; k < 3; ++k) memcpy(v[k], P[idx[k]], sizeof(float[4]));
    if (!clip_setup(sc, (const float(*)[4])v, &s[j])) continue;
    for (int k = 0; k < 3; ++k) memcpy(s[j].c[k], C[idx[s[j].vi[k]]], sizeof(float[4]));
    alive[j] = 1;
    ++m;
  }
  return m;
}

/* Raster stage: does any edge reject the tile (all 4 corner samples strictly outside)? */
static int tile_rejected(const rsetup* s, int tx, int ty) {
  int64_t x0 = tx * 8, x1 = tx * 8 + 7, y0 = ty * 8, y1 = ty * 8 + 7;
  if (x0 < s->px0) x0 = s->px0;
  if (x1 > s->px1) x1 = s->px1;
  if (y0 < s->py0) y0 = s->py0;
  if (y1 > s->py1) y1 = s->py1;
  int64_t cx[2] = {x0 * 16 + 8, x1 * 16 + 8}, cy[2] = {y0 * 16 + 8, y1 * 16 + 8};
  for (int e = 0; e < 3; ++e) {
    int a = e, b = (e + 1) % 3;
    int all_out = 1;
    for (int i = 0; i < 2 && all_out; ++i)
      for (int j = 0; j < 2 && all_out; ++j)
        if (r_edge(s->X[a], s->Y[a], s->X[b], s->Y[b], cx[i], cy[j]) >= 0) all_out = 0;
    if (all_out) return 1;
  }
  return 0;
}

/* Barycentric weights (vertex order of the setup) and inside test at a pixel centre. */
static int frag_weights(const rsetup* s, int px, int py, float l[3]) {
  int64_t Px = (int64_t)px * 16 + 8, Py = (int64_t)py * 16 + 8;
  int64_t E[3];
  E[0] = r_edge(s->X[1], s->Y[1], s->X[2], s->Y[2], Px, Py); /* opposite v0 */
  E[1] = r_edge(s->X[2], s->Y[2], s->X[0], s->Y[0], Px, Py); /* opposite v1 */
  E[2] = r_edge(s->X[0], s->Y[0], s->X[1], s->Y[1], Px, Py); /* opposite v2 */
  int in0 = E[2] > 0 || (E[2] == 0 && r_owns(s->X[0], s->Y[0], s->X[1], s->Y[1]));
  int in1 = E[0] > 0 || (E[0] == 0 && r_owns(s->X[1], s->Y[1], s->X[2], s->Y[2]));
  int in2 = E[1] > 0 || (E[1] == 0 && r_owns(s->X[2], s->Y[2], s->X[0], s->Y[0]));
  if (!(in0 && in1 && in2)) return 0;
  float A = (float)s->area;
  l[0] = (float)E[0] / A;
  l[1] = (float)E[1] / A;
  l[2] = (float)E[2] / A;
  return 1;
}

static void fragment_tile(const orc_raster_scene* sc, uint32_t tri, const rsetup* s, int tx, int ty,
                          orc_raster_out* out) {
  for (int py = ty * 8; py < ty * 8 + 8; ++py)
    for (int px = tx * 8; px < tx * 8 + 8; ++px) {
      if (px < s->px0 || px > s->px1 || py < s->py0 || py > s->py1) continue;
      float l[3];
      if (!frag_weights(s, px, py, l)) continue;
      float z = l[0] * s->z[0] + l[1] * s->z[1];
      z = z + l[2] * s->z[2];
      if (!(z >= 0.0f && z <= 1.0f)) continue;
      out->n_frag_pixels++;
      uint64_t key = ((uint64_t)r_zkey(z) << 32) | tri;
      size_t p = (size_t)py * sc->W + px;
      if (key < out->key[p]) out->key[p] = key;
    }
}

static void raster_resolve(const orc_raster_scene* sc, const rsetup* setups, const uint8_t* alive,
                           orc_raster_out* out) {
  for (int py = 0; py < sc->H; ++py)
    for (int px = 0; px < sc->W; ++px) {
      size_t p = (size_t)py * sc->W + px;
      float* c = out->colour + 4 * p;
      if (out->key[p] == UINT64_MAX) {
        c[0] = c[1] = c[2] = c[3] = 0.0f;
        continue;
      }
      uint32_t tri = (uint32_t)(out->key[p] & 0xFFFFFFFFu); /* sub-triangle id in near-clip mode */
      const rsetup* s = &setups[tri];
      float l[3] = {0, 0, 0};
      if (!alive[tri] || !frag_weights(s, px, py, l)) { /* cannot happen */
        c[0] = c[1] = c[2] = c[3] = -1.0f;
        continue;
      }
      float cv[3][4];
      for (int k = 0; k < 3; ++k)
        for (int ch = 0; ch < 4; ++ch)
          cv[k][ch] = sc->near_clip ? s->c[k][ch] : sc->col[12 * (size_t)tri + 4 * s->vi[k] + ch];
      for (int ch = 0; ch < 3; ++ch) {
        float v = l[0] * cv[0][ch] + l[1] * cv[1][ch];
        v = v + l[2] * cv[2][ch];
        c[ch] = v;
      }
      c[3] = 1.0f;
    }
}

static void raster_out_reset(const orc_raster_scene* sc, orc_raster_out* out) {
  size_t npix = (size_t)sc->W * sc->H;
  for (size_t i = 0; i < npix; ++i) out->key[i] = UINT64_MAX;
  out->n_vertex = out->n_clip = out->n_raster = out->n_fragment = out->n_frag_pixels = 0;
}

/* ---------- definition oracle: per-triangle loop into a z-buffer ---------- */
int orc_raster_definition(const orc_raster_scene* sc, orc_raster_out* out) {
  raster_out_reset(sc, out);
  const size_t nsub = (size_t)sc->n_tris * (sc->near_clip ? 2 : 1);
  rsetup* setups = (rsetup*)calloc(nsub, sizeof(rsetup));
  uint8_t* alive = (uint8_t*)calloc(nsub, 1);
  if (!setups || !alive) return 1;
  for (int64_t t = 0; t < sc->n_tris; ++t) {
    float clip[3][4];
    out->n_vertex++;
    orc_raster_vertex(sc, (uint32_t)t, clip);
    out->n_clip++;
    uint32_t ids[2];
    int m = 0;
    if (sc->near_clip) {
      int al[2];
      near_clip_setup(sc, (uint32_t)t, clip, &setups[2 * t], al);
      for (int j = 0; j < 2; ++j)
        if (al[j]) alive[2 * t + j] = 1, ids[m++] = (uint32_t)(2 * t + j);
    } else if (clip_setup(sc, clip, &setups[t])) {
      alive[t] = 1;
      ids[m++] = (uint32_t)t;
    }
    for (int i = 0; i < m; ++i) {
      out->n_raster++;
      const rsetup* s = &setups[ids[i]];
      for (int ty = s->py0 >> 3; ty <= s->py1 >> 3; ++ty)
        for (int tx = s->px0 >> 3; tx <= s->px1 >> 3; ++tx) {
          if (tile_rejected(s, tx, ty)) continue;
          out->n_fragment++;
          fragment_tile(sc, ids[i], s, tx, ty, out);
        }
    }
  }
  raster_resolve(sc, setups, alive, out);
  free(setups);
  free(alive);
  return 0;
}

/* ---------- pipeline oracle: Vertex(0) / Clip(1) / Raster(2) / Fragment(3) ---------- */
typedef struct raster_user {
  const orc_raster_scene* sc;
  orc_raster_out* out;
  float (*clip)[3][4];
  rsetup* setups;
  uint8_t* alive;
} raster_user;

static void raster_exec(orc_engine* e, int stage, const void* item) {
  raster_user* u = (raster_user*)e->user;
  if (stage < 3) {
    uint32_t tri;
    memcpy(&tri, item, 4);
    orc_record(e, stage, tri);
    if (stage == 0) {
      orc_raster_vertex(u->sc, tri, u->clip[tri]);
      orc_push(e, 1, &tri);
    } else if (stage == 1) {
      if (u->sc->near_clip) {
        int al[2];
        near_clip_setup(u->sc, tri, (const float(*)[4])u->clip[tri], &u->setups[2 * (size_t)tri], al);
        for (int j = 0; j < 2; ++j)
          if (al[j]) {
            uint32_t sub = 2 * tri + (uint32_t)j;
            u->alive[sub] = 1;
            orc_push(e, 2, &sub);
          }
      } else if (clip_setup(u->sc, (const float(*)[4])u->clip[tri], &u->setups[tri])) {
        u->alive[tri] = 1;
        orc_push(e, 2, &tri);
      }
    } else {
      const rsetup* s = &u->setups[tri];
      for (int ty = s->py0 >> 3; ty <= s->py1 >> 3; ++ty)
        for (int tx = s->px0 >> 3; tx <= s->px1 >> 3; ++tx) {
          if (tile_rejected(s, tx, ty)) continue;
          uint32_t it[2] = {tri, ((uint32_t)ty << 16) | (uint32_t)tx};
          orc_push(e, 3, it);
        }
    }
  } else {
    uint32_t it[2];
    memcpy(it, item, 8);
    orc_record(e, 3, ((uint64_t)it[0] << 32) | it[1]);
    fragment_tile(u->sc, it[0], &u->setups[it[0]], (int)(it[1] & 0xFFFF), (int)(it[1] >> 16), u->out);
  }
}

int orc_raster_pipeline(const orc_raster_scene* sc, orc_raster_out* out) {
  raster_out_reset(sc, out);
  raster_user u;
  u.sc = sc;
  u.out = out;
  u.clip = (float(*)[3][4])calloc((size_t)sc->n_tris, sizeof(float[3][4]));
  const size_t nsub = (size_t)sc->n_tris * (sc->near_clip ? 2 : 1);
  u.setups = (rsetup*)calloc(nsub, sizeof(rsetup));
  u.alive = (uint8_t*)calloc(nsub, 1);
  if (!u.clip || !u.setups || !u.alive) return 1;
  size_t strides[4] = {4, 4, 4, 8};
  orc_engine e;
  orc_engine_init(&e, 4, strides, raster_exec, &u);
  e.trace = out->trace;
  e.trace_cap = out->trace_cap;
  for (int64_t t = 0; t < sc->n_tris; ++t) {
    uint32_t tri = (uint32_t)t;
    orc_push(&e, 0, &tri);
  }
  int rc = orc_run(&e);
  out->n_vertex = e.deq[0];
  out->n_clip = e.deq[1];
  out->n_raster = e.deq[2];
  out->n_fragment = e.deq[3];
  out->trace_n = e.trace_n;
  orc_engine_free(&e);
  raster_resolve(sc, u.setups, u.alive, out);
  free(u.clip);
  free(u.setups);
  free(u.alive);
  return rc;
}

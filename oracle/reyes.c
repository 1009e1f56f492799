/* reyes.c — CPU ORACLE (test infrastructure only): Reyes rendering.
 *
 * PAPER.md L3 (Fig. 1): "Primitives -> Bound -> (diceable? N: Split -> back to Bound,
 * Y: Dice) -> Shade -> Image"; L5 "It uses one recursive stage and three other stages";
 * L55 Reyes discussion; Table 2 (L51) 272-B item.  The paper gives no formulas, so the
 * arithmetic follows SURVEY §8(c-1) with the readings listed in DESIGN.md §2 (R-R1..R-R12):
 *
 *  project:   c = M.p, row r = ((M[r0]x + M[r1]y) + M[r2]z) + M[r3]w
 *             sx = (c.x/c.w*0.5+0.5)*W, sy = (c.y/c.w*0.5+0.5)*H, zs = c.z/c.w
 *  Bound:     all c.w <= near -> cull; any c.w <= near -> cull at Dmax else split
 *             (object-space metric); bbox of the 16 (sx,sy) misses [0,W)x[0,H) -> cull;
 *             diceable iff max(bw,bh) <= T_dice or depth == Dmax.
 *  Split dir: L_u = max_b(|sx[3][b]-sx[0][b]| + |sy[3][b]-sy[0][b]|), L_v likewise
 *             along b; split u iff L_u >= L_v (tie -> u).
 *  Split:     de Casteljau at t = 1/2 on the 4 curves along that direction.
 *  Dice:      (G+1)^2 = 81 points, separable Bernstein evaluation (v-sums over b into
 *             the u-curve points C_a(v_j), then u-sums over a), project.
 *  Shade:     per micropolygon q = (i,j): n = cross(p10-p00, p01-p00),
 *             s = 0.1 + 0.9*max(0, n.L/|n|) (0.1 if |n| = 0); coverage of the two
 *             triangles (v00,v10,v11), (v00,v11,v01) at pixel centres, Q8 fixed point,
 *             int64 edge functions, top-left-style fill rule; flat depth
 *             zq = ((z00+z10)+(z11+z01))*0.25; per pixel keep min (zkey(zq) << 32 | mp_id).
 *  Resolve:   colour = albedo[patch] * s (alpha 1) for covered pixels, 0 otherwise.
 *
 * Two oracles: orc_reyes_definition (textbook DFS recursion, Cook et al. [12]) and
 * orc_reyes_pipeline (the fixpoint engine over Bound/Split/Dice/Shade queues).
 */
#include <math.h>
#include <stdlib.h>
#include <string.h>

#include "oracle.h"

#define G 8
#define NG (G + 1)

void orc_reyes_project(const float M[16], const float p[4], float c[4]) {
  for (int r = 0; r < 4; ++r) {
    float acc = M[4 * r + 0] * p[0];
    acc = acc + M[4 * r + 1] * p[1];
    acc = acc + M[4 * r + 2] * p[2];
    acc = acc + M[4 * r + 3] * p[3];
    c[r] = acc;
  }
}

static void to_screen(const orc_reyes_scene* sc, const float c[4], float* sx, float* sy, float* zs) {
  float nx = c[0] / c[3];
  float ny = c[1] / c[3];
  *sx = (nx * 0.5f + 0.5f) * (float)sc->W;
  *sy = (ny * 0.5f + 0.5f) * (float)sc->H;
  *zs = c[2] / c[3];
}

static const float* frame_M(const orc_reyes_scene* sc, uint32_t id) {
  return sc->M + 16 * (size_t)(id >> 12);
}

/* Bound (Fig. 1 "Bound" + "diceable?"): returns ORC_REYES_{CULL,SPLIT,DICE}. */
int orc_reyes_bound(const orc_reyes_scene* sc, const orc_patch* p, int* split_dir) {
  const float* M = frame_M(sc, p->id);
  float c[16][4];
  int n_behind = 0;
  for (int k = 0; k < 16; ++k) {
    orc_reyes_project(M, p->cp[k], c[k]);
    if (!(c[k][3] > sc->near_w)) n_behind++;
  }
  *split_dir = 0;
  if (n_behind == 16) return ORC_REYES_CULL;
  if (n_behind > 0) {
    /* straddles the near plane: cannot bound in screen space (reading R-R4) */
    if ((int)p->depth >= sc->max_depth) return ORC_REYES_CULL;
    float Lu = 0.0f, Lv = 0.0f;
    for (int b = 0; b < 4; ++b) {
      const float* a0 = p->cp[0 * 4 + b];
      const float* a3 = p->cp[3 * 4 + b];
      float l = fabsf(a3[0] - a0[0]) + fabsf(a3[1] - a0[1]);
      l = l + fabsf(a3[2] - a0[2]);
      if (l > Lu) Lu = l;
    }
    for (int a = 0; a < 4; ++a) {
      const float* b0 = p->cp[a * 4 + 0];
      const float* b3 = p->cp[a * 4 + 3];
      float l = fabsf(b3[0] - b0[0]) + fabsf(b3[1] - b0[1]);
      l = l + fabsf(b3[2] - b0[2]);
      if (l > Lv) Lv = l;
    }
    *split_dir = (Lu >= Lv) ? 0 : 1;
    return ORC_REYES_SPLIT;
  }
  float sx[16], sy[16], zs;
  for (int k = 0; k < 16; ++k) to_screen(sc, c[k], &sx[k], &sy[k], &zs);
  float xmin = sx[0], xmax = sx[0], ymin = sy[0], ymax = sy[0];
  for (int k = 1; k < 16; ++k) {
    if (sx[k] < xmin) xmin = sx[k];
    if (sx[k] > xmax) xmax = sx[k];
    if (sy[k] < ymin) ymin = sy[k];
    if (sy[k] > ymax) ymax = sy[k];
  }
  if (xmax < 0.0f || xmin >= (float)sc->W || ymax < 0.0f || ymin >= (float)sc->H) return ORC_REYES_CULL;
  float bw = xmax - xmin, bh = ymax - ymin;
  float ext = bw > bh ? bw : bh;
  if ((int)p->depth >= sc->max_depth || ext <= sc->t_dice) return ORC_REYES_DICE;
  float Lu = 0.0f, Lv = 0.0f;
  for (int b = 0; b < 4; ++b) {
    float l = fabsf(sx[12 + b] - sx[b]) + fabsf(sy[12 + b] - sy[b]);
    if (l > Lu) Lu = l;
  }
  for (int a = 0; a < 4; ++a) {
    float l = fabsf(sx[4 * a + 3] - sx[4 * a]) + fabsf(sy[4 * a + 3] - sy[4 * a]);
    if (l > Lv) Lv = l;
  }
  *split_dir = (Lu >= Lv) ? 0 : 1;
  return ORC_REYES_SPLIT;
}

/* de Casteljau at t = 1/2 (reading R-R6), exactly this operation order. */
static void casteljau(float a, float b, float c, float d, float L[4], float R[4]) {
  float ab = (a + b) * 0.5f, bc = (b + c) * 0.5f, cd = (c + d) * 0.5f;
  float abc = (ab + bc) * 0.5f, bcd = (bc + cd) * 0.5f;
  float m = (abc + bcd) * 0.5f;
  L[0] = a; L[1] = ab; L[2] = abc; L[3] = m;
  R[0] = m; R[1] = bcd; R[2] = cd; R[3] = d;
}

void orc_reyes_split(const orc_patch* p, int dir, orc_patch* left, orc_patch* right) {
  *left = *p;
  *right = *p;
  for (int line = 0; line < 4; ++line) {
    int idx[4];
    for (int t = 0; t < 4; ++t) idx[t] = (dir == 0) ? (4 * t + line) : (4 * line + t);
    for (int comp = 0; comp < 4; ++comp) {
      float Lc[4], Rc[4];
      casteljau(p->cp[idx[0]][comp], p->cp[idx[1]][comp], p->cp[idx[2]][comp], p->cp[idx[3]][comp], Lc, Rc);
      for (int t = 0; t < 4; ++t) {
        left->cp[idx[t]][comp] = Lc[t];
        right->cp[idx[t]][comp] = Rc[t];
      }
    }
  }
  uint32_t d = p->depth;
  left->depth = right->depth = d + 1;
  left->dirs = right->dirs = (p->dirs & ~(1u << d)) | ((uint32_t)dir << d);
  left->path = p->path & ~(1u << d);
  right->path = p->path | (1u << d);
}

static void bernstein(float t, float B[4]) {
  float s = 1.0f - t;
  B[0] = (s * s) * s;
  B[1] = ((3.0f * t) * s) * s;
  B[2] = ((3.0f * t) * t) * s;
  B[3] = (t * t) * t;
}

/* Dice: grid[0..5][g], g = i*9 + j, rows x,y,z (object) and sx,sy,zs (screen).
 * Reading R-R7: the tensor-product Bezier surface S(u,v) = sum_a B_a(u) sum_b B_b(v) P_ab
 * evaluated in its separable (two-stage) form at u_i = i/8, v_j = j/8: first the four
 * u-curve control points at v_j, C_a(v_j) = sum_b B_b(v_j) P_ab (b = 0..3 in order), then
 * S(u_i, v_j) = sum_a B_a(u_i) C_a(v_j) (a = 0..3 in order); every sum starts at 0. */
void orc_reyes_dice(const orc_reyes_scene* sc, const orc_patch* p, float grid[6][81]) {
  const float* M = frame_M(sc, p->id);
  float C[4][NG][3];
  for (int a = 0; a < 4; ++a)
    for (int j = 0; j < NG; ++j) {
      float Bv[4];
      bernstein((float)j * 0.125f, Bv);
      for (int k = 0; k < 3; ++k) {
        float acc = 0.0f;
        for (int b = 0; b < 4; ++b) acc = acc + Bv[b] * p->cp[4 * a + b][k];
        C[a][j][k] = acc;
      }
    }
  for (int i = 0; i < NG; ++i) {
    float Bu[4];
    bernstein((float)i * 0.125f, Bu);
    for (int j = 0; j < NG; ++j) {
      float xyz[3];
      for (int k = 0; k < 3; ++k) {
        float acc = 0.0f;
        for (int a = 0; a < 4; ++a) acc = acc + Bu[a] * C[a][j][k];
        xyz[k] = acc;
      }
      const float x = xyz[0], y = xyz[1], z = xyz[2];
      float q[4] = {x, y, z, 1.0f}, c[4];
      orc_reyes_project(M, q, c);
      int g = i * NG + j;
      grid[0][g] = x;
      grid[1][g] = y;
      grid[2][g] = z;
      to_screen(sc, c, &grid[3][g], &grid[4][g], &grid[5][g]);
    }
  }
}

float orc_reyes_shade_factor(const float n[3], const float L[4]) {
  float nn = n[0] * n[0] + n[1] * n[1];
  nn = nn + n[2] * n[2];
  if (nn == 0.0f) return 0.1f;
  float d = n[0] * L[0] + n[1] * L[1];
  d = d + n[2] * L[2];
  float t = d / sqrtf(nn);
  if (!(t > 0.0f)) t = 0.0f;
  return 0.1f + 0.9f * t;
}

static uint32_t zkey(float z) {
  uint32_t b;
  memcpy(&b, &z, 4);
  return (b & 0x80000000u) ? ~b : (b | 0x80000000u);
}

static int64_t floor_div256(int64_t a) { return a >= 0 ? a / 256 : -((-a + 255) / 256); }
static int64_t ceil_div256(int64_t a) { return -floor_div256(-a); }

static int64_t edge_fn(const int64_t* a, const int64_t* b, int64_t px, int64_t py) {
  return (b[0] - a[0]) * (py - a[1]) - (b[1] - a[1]) * (px - a[0]);
}

/* edge a->b of a positively oriented triangle owns its boundary points iff
 * dy > 0 || (dy == 0 && dx < 0)  (reading R-R9; equals sampling at P - (eps, eps^2)) */
static int owned(const int64_t* a, const int64_t* b) {
  int64_t dx = b[0] - a[0], dy = b[1] - a[1];
  return dy > 0 || (dy == 0 && dx < 0);
}

static void raster_tri(const orc_reyes_scene* sc, uint64_t* fbkey, float* fbs, const int64_t* v0, const int64_t* v1,
                       const int64_t* v2, uint64_t key, float s) {
  const int64_t* a = v0;
  const int64_t* b = v1;
  const int64_t* c = v2;
  int64_t area = edge_fn(a, b, c[0], c[1]);
  if (area == 0) return;
  if (area < 0) { const int64_t* t = b; b = c; c = t; }
  int64_t xmin = a[0], xmax = a[0], ymin = a[1], ymax = a[1];
  const int64_t* vs[2] = {b, c};
  for (int k = 0; k < 2; ++k) {
    if (vs[k][0] < xmin) xmin = vs[k][0];
    if (vs[k][0] > xmax) xmax = vs[k][0];
    if (vs[k][1] < ymin) ymin = vs[k][1];
    if (vs[k][1] > ymax) ymax = vs[k][1];
  }
  int64_t px0 = ceil_div256(xmin - 128), px1 = floor_div256(xmax - 128);
  int64_t py0 = ceil_div256(ymin - 128), py1 = floor_div256(ymax - 128);
  if (px0 < 0) px0 = 0;
  if (py0 < 0) py0 = 0;
  if (px1 > sc->W - 1) px1 = sc->W - 1;
  if (py1 > sc->H - 1) py1 = sc->H - 1;
  for (int64_t py = py0; py <= py1; ++py)
    for (int64_t px = px0; px <= px1; ++px) {
      int64_t X = px * 256 + 128, Y = py * 256 + 128;
      int64_t w0 = edge_fn(a, b, X, Y), w1 = edge_fn(b, c, X, Y), w2 = edge_fn(c, a, X, Y);
      int in0 = w0 > 0 || (w0 == 0 && owned(a, b));
      int in1 = w1 > 0 || (w1 == 0 && owned(b, c));
      int in2 = w2 > 0 || (w2 == 0 && owned(c, a));
      if (in0 && in1 && in2) {
        size_t pix = (size_t)py * sc->W + (size_t)px;
        if (key < fbkey[pix]) {
          fbkey[pix] = key;
          fbs[pix] = s;
        }
      }
    }
}

/* Shade one diced grid into the frame's key/s buffers (Fig. 1 "Shade" -> "Image"). */
static void shade_grid(const orc_reyes_scene* sc, uint32_t id, uint32_t path, uint32_t depth, const float grid[6][81],
                       uint64_t* key_all, float* s_all, uint64_t* n_covering) {
  size_t frame = id >> 12;
  uint32_t patch = id & 0xFFFu;
  uint64_t* fbkey = key_all + frame * (size_t)sc->W * sc->H;
  float* fbs = s_all + frame * (size_t)sc->W * sc->H;
  for (int i = 0; i < G; ++i)
    for (int j = 0; j < G; ++j) {
      int g00 = i * NG + j, g10 = (i + 1) * NG + j, g01 = i * NG + j + 1, g11 = (i + 1) * NG + j + 1;
      float e1[3], e2[3], n[3];
      for (int k = 0; k < 3; ++k) {
        e1[k] = grid[k][g10] - grid[k][g00];
        e2[k] = grid[k][g01] - grid[k][g00];
      }
      n[0] = e1[1] * e2[2] - e1[2] * e2[1];
      n[1] = e1[2] * e2[0] - e1[0] * e2[2];
      n[2] = e1[0] * e2[1] - e1[1] * e2[0];
      float s = orc_reyes_shade_factor(n, sc->L);
      float zq = ((grid[5][g00] + grid[5][g10]) + (grid[5][g11] + grid[5][g01])) * 0.25f;
      uint32_t q = (uint32_t)(i * G + j);
      uint32_t mp = (patch << 18) | ((path & 0xFFu) << 10) | ((depth & 0xFu) << 6) | q;
      uint64_t key = ((uint64_t)zkey(zq) << 32) | mp;
      int gi[4] = {g00, g10, g11, g01};
      int64_t v[4][2];
      int ok = 1;
      for (int k = 0; k < 4; ++k) {
        float X = grid[3][gi[k]] * 256.0f, Y = grid[4][gi[k]] * 256.0f;
        if (!(fabsf(X) < 1073741824.0f) || !(fabsf(Y) < 1073741824.0f)) ok = 0;
        else {
          v[k][0] = (int64_t)rintf(X);
          v[k][1] = (int64_t)rintf(Y);
        }
      }
      if (!ok) continue;
      {  /* does the quad's box hold a pixel centre (px + 0.5, py + 0.5) on the screen? */
        int64_t xmin = v[0][0], xmax = v[0][0], ymin = v[0][1], ymax = v[0][1];
        for (int k = 1; k < 4; ++k) {
          if (v[k][0] < xmin) xmin = v[k][0];
          if (v[k][0] > xmax) xmax = v[k][0];
          if (v[k][1] < ymin) ymin = v[k][1];
          if (v[k][1] > ymax) ymax = v[k][1];
        }
        int64_t px0 = ceil_div256(xmin - 128), px1 = floor_div256(xmax - 128);
        int64_t py0 = ceil_div256(ymin - 128), py1 = floor_div256(ymax - 128);
        if (px0 < 0) px0 = 0;
        if (py0 < 0) py0 = 0;
        if (px1 > sc->W - 1) px1 = sc->W - 1;
        if (py1 > sc->H - 1) py1 = sc->H - 1;
        if (px0 <= px1 && py0 <= py1) ++*n_covering;
      }
      raster_tri(sc, fbkey, fbs, v[0], v[1], v[2], key, s);
      raster_tri(sc, fbkey, fbs, v[0], v[2], v[3], key, s);
    }
}

static void reyes_out_reset(const orc_reyes_scene* sc, orc_reyes_out* out) {
  size_t npix = (size_t)sc->n_frames * sc->W * sc->H;
  for (size_t i = 0; i < npix; ++i) {
    out->key[i] = UINT64_MAX;
    out->s[i] = 0.0f;
  }
  out->n_bound = out->n_split = out->n_dice = out->n_shade = out->n_culled = 0;
  out->n_mp_covering = 0;
  memset(out->depth_hist, 0, sizeof(out->depth_hist));
  memset(out->culled_depth_hist, 0, sizeof(out->culled_depth_hist));
  out->n_leaves = 0;
  out->trace_n = 0;
}

static void resolve(const orc_reyes_scene* sc, orc_reyes_out* out) {
  size_t npix = (size_t)sc->W * sc->H;
  for (size_t f = 0; f < (size_t)sc->n_frames; ++f)
    for (size_t p = 0; p < npix; ++p) {
      size_t i = f * npix + p;
      float* c = out->colour + 4 * i;
      if (out->key[i] == UINT64_MAX) {
        c[0] = c[1] = c[2] = c[3] = 0.0f;
      } else {
        uint32_t patch = (uint32_t)(out->key[i] >> 18) & 0xFFFu;
        const float* alb = sc->albedo + 4 * (size_t)patch;
        c[0] = alb[0] * out->s[i];
        c[1] = alb[1] * out->s[i];
        c[2] = alb[2] * out->s[i];
        c[3] = 1.0f;
      }
    }
}

static uint64_t node_id(const orc_patch* p) {
  return ((uint64_t)p->id << 12) | ((uint64_t)(p->depth & 0xF) << 8) | (p->path & 0xFF);
}

static void record_leaf(orc_reyes_out* out, const orc_patch* p, float grid[6][81]) {
  if (out->leaf_ids && out->n_leaves < out->leaf_cap) {
    out->leaf_ids[out->n_leaves] = node_id(p);
    if (out->leaf_grids) memcpy(out->leaf_grids + out->n_leaves * 6 * 81, grid, sizeof(float) * 6 * 81);
  }
  out->n_leaves++;
}

/* ---------- definition oracle: textbook depth-first recursion ---------- */
static void visit(const orc_reyes_scene* sc, const orc_patch* p, orc_reyes_out* out) {
  out->n_bound++;
  int dir;
  int cls = orc_reyes_bound(sc, p, &dir);
  if (cls == ORC_REYES_CULL) {
    out->n_culled++;
    out->culled_depth_hist[p->depth & 15]++;
  } else if (cls == ORC_REYES_DICE) {
    float grid[6][81];
    out->n_dice++;
    out->n_shade++;
    out->depth_hist[p->depth & 15]++;
    orc_reyes_dice(sc, p, grid);
    record_leaf(out, p, grid);
    shade_grid(sc, p->id, p->path, p->depth, (const float(*)[81])grid, out->key, out->s, &out->n_mp_covering);
  } else {
    orc_patch l, r;
    out->n_split++;
    orc_reyes_split(p, dir, &l, &r);
    visit(sc, &l, out);
    visit(sc, &r, out);
  }
}

int orc_reyes_definition(const orc_reyes_scene* sc, const orc_patch* seeds, size_t n, orc_reyes_out* out) {
  reyes_out_reset(sc, out);
  for (size_t i = 0; i < n; ++i) visit(sc, &seeds[i], out);
  resolve(sc, out);
  return 0;
}

/* ---------- pipeline oracle: Bound(0) / Split(1) / Dice(2) / Shade(3) queues ---------- */
typedef struct reyes_grid_item {
  uint32_t id, path, depth, dirs;
  float grid[6][81];
} reyes_grid_item;

typedef struct reyes_user {
  const orc_reyes_scene* sc;
  orc_reyes_out* out;
} reyes_user;

static void reyes_exec(orc_engine* e, int stage, const void* item) {
  reyes_user* u = (reyes_user*)e->user;
  if (stage == 0) { /* Bound */
    orc_patch p;
    memcpy(&p, item, sizeof(p));
    orc_record(e, 0, node_id(&p));
    int dir;
    int cls = orc_reyes_bound(u->sc, &p, &dir);
    if (cls == ORC_REYES_CULL) {
      u->out->n_culled++;
      u->out->culled_depth_hist[p.depth & 15]++;
    } else if (cls == ORC_REYES_DICE) {
      orc_push(e, 2, &p);
    } else {
      p.dirs = (p.dirs & ~(1u << p.depth)) | ((uint32_t)dir << p.depth);
      orc_push(e, 1, &p);
    }
  } else if (stage == 1) { /* Split */
    orc_patch p, l, r;
    memcpy(&p, item, sizeof(p));
    orc_record(e, 1, node_id(&p));
    orc_reyes_split(&p, (int)((p.dirs >> p.depth) & 1u), &l, &r);
    orc_push(e, 0, &l);
    orc_push(e, 0, &r);
  } else if (stage == 2) { /* Dice */
    orc_patch p;
    memcpy(&p, item, sizeof(p));
    orc_record(e, 2, node_id(&p));
    reyes_grid_item gi;
    gi.id = p.id;
    gi.path = p.path;
    gi.depth = p.depth;
    gi.dirs = p.dirs;
    orc_reyes_dice(u->sc, &p, gi.grid);
    u->out->depth_hist[p.depth & 15]++;
    record_leaf(u->out, &p, gi.grid);
    orc_push(e, 3, &gi);
  } else { /* Shade */
    const reyes_grid_item* gi = (const reyes_grid_item*)item;
    orc_record(e, 3, ((uint64_t)gi->id << 12) | ((uint64_t)(gi->depth & 0xF) << 8) | (gi->path & 0xFF));
    shade_grid(u->sc, gi->id, gi->path, gi->depth, (const float(*)[81])gi->grid, u->out->key, u->out->s,
               &u->out->n_mp_covering);
  }
}

int orc_reyes_pipeline(const orc_reyes_scene* sc, const orc_patch* seeds, size_t n, orc_reyes_out* out) {
  reyes_out_reset(sc, out);
  size_t strides[4] = {sizeof(orc_patch), sizeof(orc_patch), sizeof(orc_patch), sizeof(reyes_grid_item)};
  reyes_user u = {sc, out};
  orc_engine e;
  orc_engine_init(&e, 4, strides, reyes_exec, &u);
  e.trace = out->trace;
  e.trace_cap = out->trace_cap;
  for (size_t i = 0; i < n; ++i) orc_push(&e, 0, &seeds[i]);
  int rc = orc_run(&e);
  out->n_bound = e.deq[0];
  out->n_split = e.deq[1];
  out->n_dice = e.deq[2];
  out->n_shade = e.deq[3];
  out->trace_n = e.trace_n;
  orc_engine_free(&e);
  resolve(sc, out);
  return rc;
}

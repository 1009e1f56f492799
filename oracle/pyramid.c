/* pyramid.c — CPU ORACLE (test infrastructure only): image pyramid.
 *
 * PAPER.md L53 (Fig. 12: Grayscale -> Histogram Equalization -> Resize, recursive),
 * Table 1 L43 (3 stages, recursion, dynamic), L51 (12-B items; HistEq's serial part is
 * 96.1% of KBK time), L55 (HistEq split into 3 kernels in KBK).  The paper gives no
 * formulas; DESIGN.md §2 readings R-P1..R-P6:
 *
 *  Grayscale:  Y = (77 R + 150 G + 29 B + 128) >> 8.
 *  HistEq:     hist over the N level-0 pixels, cdf, cmin = cdf at the first non-empty
 *              bin; LUT[v] = ((cdf[v]-cmin)*255 + (N-cmin)/2) / (N-cmin) (integer), 0
 *              below the first non-empty bin; identity if N == cmin.  Level 0 = LUT[Y].
 *  Resize:     level l+1 = 2x2 box of level l: (a+b+c+d+2) >> 2, down to 1x1.
 *
 * Pipeline decomposition (R-P4): Gray(tile 64x64) -> [latch: all level-0 tiles of an
 * image] -> CDF(image) -> Map(image, 8-tile row segment) -> [latch per level-1 tile]
 * -> Resize(level, tile) -> [latch per next-level tile] -> ... (dependency latches,
 * SURVEY §8(a) row a8).
 */
#include <stdlib.h>
#include <string.h>

#include "oracle.h"

#define PT 64   /* tile side */
#define MAPSEG 8 /* level-0 tiles per Map item */

static int lvl_size(const orc_pyr_scene* sc, int l) { return sc->S >> l; }
static int lvl_tiles(const orc_pyr_scene* sc, int l) {
  int s = lvl_size(sc, l);
  return s >= PT ? s / PT : 1;
}
int orc_pyr_levels(int S) {
  int L = 0;
  while ((S >> L) >= 1) ++L;
  return L; /* levels 0..L-1, last one 1x1 */
}
size_t orc_pyr_level_offset(int S, int l) {
  size_t off = 0;
  for (int k = 0; k < l; ++k) off += (size_t)(S >> k) * (size_t)(S >> k);
  return off;
}

static uint8_t gray_px(const uint8_t* rgb) {
  return (uint8_t)((77u * rgb[0] + 150u * rgb[1] + 29u * rgb[2] + 128u) >> 8);
}

void orc_histeq_lut(const uint32_t hist[256], uint64_t N, uint8_t lut[256]) {
  uint64_t cdf[256], acc = 0;
  int first = -1;
  for (int v = 0; v < 256; ++v) {
    acc += hist[v];
    cdf[v] = acc;
    if (first < 0 && hist[v]) first = v;
  }
  uint64_t cmin = first >= 0 ? cdf[first] : 0;
  for (int v = 0; v < 256; ++v) {
    if (N == cmin) lut[v] = (uint8_t)v;
    else if (v < first) lut[v] = 0;
    else lut[v] = (uint8_t)(((cdf[v] - cmin) * 255u + (N - cmin) / 2u) / (N - cmin));
  }
}

/* 2x2 box of one output pixel (x, y) of level l (>= 1) from level l-1 */
static uint8_t box(const orc_pyr_scene* sc, const uint8_t* pyr_img, int l, int x, int y) {
  int sp = lvl_size(sc, l - 1);
  const uint8_t* src = pyr_img + orc_pyr_level_offset(sc->S, l - 1);
  unsigned a = src[(size_t)(2 * y) * sp + 2 * x], b = src[(size_t)(2 * y) * sp + 2 * x + 1];
  unsigned c = src[(size_t)(2 * y + 1) * sp + 2 * x], d = src[(size_t)(2 * y + 1) * sp + 2 * x + 1];
  return (uint8_t)((a + b + c + d + 2u) >> 2);
}

static void out_reset(const orc_pyr_scene* sc, orc_pyr_out* out) {
  memset(out->hist, 0, sizeof(uint32_t) * 256 * (size_t)sc->n_img);
  out->n_gray = out->n_cdf = out->n_map = out->n_resize = 0;
  out->trace_n = 0;
}

/* ---------- definition oracle: whole-image loops, level by level ---------- */
int orc_pyr_definition(const orc_pyr_scene* sc, orc_pyr_out* out) {
  out_reset(sc, out);
  const int S = sc->S, L = orc_pyr_levels(S);
  const size_t npx = (size_t)S * S, total = orc_pyr_level_offset(S, L);
  for (int i = 0; i < sc->n_img; ++i) {
    const uint8_t* rgb = sc->rgb + (size_t)i * npx * 3;
    uint8_t* gray = out->gray + (size_t)i * npx;
    uint32_t* hist = out->hist + 256 * (size_t)i;
    for (size_t p = 0; p < npx; ++p) {
      gray[p] = gray_px(rgb + 3 * p);
      hist[gray[p]]++;
    }
    uint8_t* lut = out->lut + 256 * (size_t)i;
    orc_histeq_lut(hist, npx, lut);
    uint8_t* pyr = out->pyr + (size_t)i * total;
    for (size_t p = 0; p < npx; ++p) pyr[p] = lut[gray[p]];
    for (int l = 1; l < L; ++l) {
      int s = lvl_size(sc, l);
      uint8_t* dst = pyr + orc_pyr_level_offset(S, l);
      for (int y = 0; y < s; ++y)
        for (int x = 0; x < s; ++x) dst[(size_t)y * s + x] = box(sc, pyr, l, x, y);
    }
  }
  return 0;
}

/* ---------- pipeline oracle: Gray(0) / CDF(1) / Map(2) / Resize(3) with latches ---------- */
typedef struct pyr_item { uint32_t img, level, ty, tx; } pyr_item;

typedef struct pyr_user {
  const orc_pyr_scene* sc;
  orc_pyr_out* out;
  int L;
  size_t lat_per_img;
  size_t lat_off[32]; /* latch index offset of level l (l >= 1) inside an image's block */
  int64_t* latch;      /* [n_img][1 + sum_{l>=1} tiles_l^2]: [0] = CDF latch */
} pyr_user;

static int64_t* resize_latch(pyr_user* u, uint32_t img, int l, int ty, int tx) {
  int nt = lvl_tiles(u->sc, l);
  return &u->latch[img * u->lat_per_img + u->lat_off[l] + (size_t)ty * nt + tx];
}

/* a finished tile (ty, tx) of level l (or k source tiles of it) arrives on level l+1 */
static void arrive_next(orc_engine* e, pyr_user* u, uint32_t img, int l, int ty, int tx, int k) {
  if (l + 1 >= u->L) return;
  int64_t* lat = resize_latch(u, img, l + 1, ty / 2, tx / 2);
  *lat -= k;
  if (*lat == 0) {
    pyr_item it = {img, (uint32_t)(l + 1), (uint32_t)(ty / 2), (uint32_t)(tx / 2)};
    orc_push(e, 3, &it);
  }
}

static void pyr_exec(orc_engine* e, int stage, const void* item) {
  pyr_user* u = (pyr_user*)e->user;
  const orc_pyr_scene* sc = u->sc;
  pyr_item it;
  memcpy(&it, item, sizeof(it));
  const int S = sc->S;
  const size_t npx = (size_t)S * S, total = orc_pyr_level_offset(S, u->L);
  orc_record(e, stage, ((uint64_t)it.img << 40) | ((uint64_t)it.level << 32) | (it.ty << 16) | it.tx);
  if (stage == 0) { /* Gray tile */
    const uint8_t* rgb = sc->rgb + (size_t)it.img * npx * 3;
    uint8_t* gray = u->out->gray + (size_t)it.img * npx;
    uint32_t* hist = u->out->hist + 256 * (size_t)it.img;
    for (int y = 0; y < PT; ++y)
      for (int x = 0; x < PT; ++x) {
        size_t p = (size_t)(it.ty * PT + y) * S + it.tx * PT + x;
        gray[p] = gray_px(rgb + 3 * p);
        hist[gray[p]]++;
      }
    int64_t* lat = &u->latch[it.img * u->lat_per_img];
    if (--*lat == 0) {
      pyr_item c = {it.img, 0, 0, 0};
      orc_push(e, 1, &c);
    }
  } else if (stage == 1) { /* CDF: LUT, then the Map items */
    orc_histeq_lut(u->out->hist + 256 * (size_t)it.img, npx, u->out->lut + 256 * (size_t)it.img);
    int nt = lvl_tiles(sc, 0);
    for (int ty = 0; ty < nt; ++ty)
      for (int seg = 0; seg < (nt + MAPSEG - 1) / MAPSEG; ++seg) {
        pyr_item m = {it.img, 0, (uint32_t)ty, (uint32_t)(seg * MAPSEG)};
        orc_push(e, 2, &m);
      }
  } else if (stage == 2) { /* Map: equalise a row segment of level-0 tiles */
    const uint8_t* lut = u->out->lut + 256 * (size_t)it.img;
    const uint8_t* gray = u->out->gray + (size_t)it.img * npx;
    uint8_t* pyr = u->out->pyr + (size_t)it.img * total;
    int nt = lvl_tiles(sc, 0);
    int tx1 = (int)it.tx + MAPSEG < nt ? (int)it.tx + MAPSEG : nt;
    for (int y = 0; y < PT; ++y)
      for (int x = (int)it.tx * PT; x < tx1 * PT; ++x) {
        size_t p = (size_t)(it.ty * PT + y) * S + x;
        pyr[p] = lut[gray[p]];
      }
    for (int tx = (int)it.tx; tx < tx1; ++tx) arrive_next(e, u, it.img, 0, (int)it.ty, tx, 1);
  } else { /* Resize: one output tile of level it.level */
    uint8_t* pyr = u->out->pyr + (size_t)it.img * total;
    int l = (int)it.level, s = lvl_size(sc, l);
    int w = s < PT ? s : PT;
    uint8_t* dst = pyr + orc_pyr_level_offset(S, l);
    for (int y = 0; y < w; ++y)
      for (int x = 0; x < w; ++x) {
        int gx = (int)it.tx * PT + x, gy = (int)it.ty * PT + y;
        dst[(size_t)gy * s + gx] = box(sc, pyr, l, gx, gy);
      }
    arrive_next(e, u, it.img, l, (int)it.ty, (int)it.tx, 1);
  }
}

int orc_pyr_pipeline(const orc_pyr_scene* sc, orc_pyr_out* out) {
  out_reset(sc, out);
  pyr_user u;
  memset(&u, 0, sizeof(u));
  u.sc = sc;
  u.out = out;
  u.L = orc_pyr_levels(sc->S);
  if (u.L > 32) return 1;
  size_t n = 1;
  for (int l = 1; l < u.L; ++l) {
    u.lat_off[l] = n;
    n += (size_t)lvl_tiles(sc, l) * lvl_tiles(sc, l);
  }
  u.lat_per_img = n;
  u.latch = (int64_t*)calloc(n * (size_t)sc->n_img, sizeof(int64_t));
  if (!u.latch) return 1;
  for (int i = 0; i < sc->n_img; ++i) {
    u.latch[i * n] = (int64_t)lvl_tiles(sc, 0) * lvl_tiles(sc, 0);
    for (int l = 1; l < u.L; ++l) {
      int src = lvl_tiles(sc, l - 1) >= 2 ? 2 : 1; /* source tiles per side in level l-1 */
      for (size_t k = 0; k < (size_t)lvl_tiles(sc, l) * lvl_tiles(sc, l); ++k)
        u.latch[i * n + u.lat_off[l] + k] = src * src;
    }
  }
  size_t strides[4] = {16, 16, 16, 16};
  orc_engine e;
  orc_engine_init(&e, 4, strides, pyr_exec, &u);
  e.trace = out->trace;
  e.trace_cap = out->trace_cap;
  int nt = lvl_tiles(sc, 0);
  for (int i = 0; i < sc->n_img; ++i)
    for (int ty = 0; ty < nt; ++ty)
      for (int tx = 0; tx < nt; ++tx) {
        pyr_item it = {(uint32_t)i, 0, (uint32_t)ty, (uint32_t)tx};
        orc_push(&e, 0, &it);
      }
  int rc = orc_run(&e);
  out->n_gray = e.deq[0];
  out->n_cdf = e.deq[1];
  out->n_map = e.deq[2];
  out->n_resize = e.deq[3];
  out->trace_n = e.trace_n;
  for (size_t k = 0; k < n * (size_t)sc->n_img; ++k)
    if (u.latch[k] != 0) rc = rc ? rc : 3; /* every latch must have fired exactly */
  orc_engine_free(&e);
  free(u.latch);
  return rc;
}

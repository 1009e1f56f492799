/* facedet.c — CPU ORACLE (test infrastructure only): LBP face detection.
 *
 * PAPER.md L55 (Fig. 14: Grayscale -> Histogram Equalization -> Resize (recursive) ->
 * Feature Extraction -> Scanning; windows without faces end early -> load imbalance; the
 * window is the data item), Table 1 L43 (5 stages, recursion, dynamic), Table 2
 * (16-B items), LBP features [2].  No trained cascade exists, so the cascade is
 * synthetic.  Readings (R-D1..R-D8):
 *  Gray      Y = (77R + 150G + 29B + 128) >> 8                      (as the pyramid)
 *  HistEq    the pyramid's LUT on level 0
 *  Resize    W' = floor(4W/5), H' = floor(4H/5), dst(x,y) = src((5x)>>2, (5y)>>2), 8
 *            levels (fewer if a side drops below 24)
 *  LBP_8,1   neighbours (-1,-1),(0,-1),(1,-1),(1,0),(1,1),(0,1),(-1,1),(-1,0) -> bits
 *            0..7, bit set iff g_p >= g_c; border pixels code 0
 *  Scan      24x24 windows, stride 1, all levels; K = 12 stages, stage k has 2+k weak
 *            classifiers {cx, cy in [1,22], mask[8], in, out}; s_k = sum(bit ? in : out);
 *            pass iff s_k >= thr_k; a window passing all stages is a detection.
 * Pipeline decomposition (R-D6): 32-row bands; latches per (level, band) for Resize and
 * LBP and per (level, window-row group) for Scan; Scan items are rows of windows
 * (composite items, L37).
 */
#include <stdlib.h>
#include <string.h>

#include "oracle.h"

#define BAND 32
#define WIN 24

static uint8_t fd_gray(const uint8_t* rgb) {
  return (uint8_t)((77u * rgb[0] + 150u * rgb[1] + 29u * rgb[2] + 128u) >> 8);
}

int orc_fd_levels(int W, int H, int* Ws, int* Hs) {
  int L = 0, w = W, h = H;
  while (L < 8 && w >= WIN && h >= WIN) {
    Ws[L] = w;
    Hs[L] = h;
    ++L;
    w = (4 * w) / 5;
    h = (4 * h) / 5;
  }
  return L;
}

static size_t lvl_off(const int* Ws, const int* Hs, int l) {
  size_t o = 0;
  for (int k = 0; k < l; ++k) o += (size_t)Ws[k] * Hs[k];
  return o;
}

static uint8_t lbp_at(const uint8_t* img, int W, int H, int x, int y) {
  if (x <= 0 || y <= 0 || x >= W - 1 || y >= H - 1) return 0;
  static const int dx[8] = {-1, 0, 1, 1, 1, 0, -1, -1}, dy[8] = {-1, -1, -1, 0, 1, 1, 1, 0};
  uint8_t c = img[(size_t)y * W + x], code = 0;
  for (int p = 0; p < 8; ++p)
    if (img[(size_t)(y + dy[p]) * W + x + dx[p]] >= c) code |= (uint8_t)(1u << p);
  return code;
}

/* cascade: weak classifier w = [cx, cy, mask0..7, in, out] (12 int32) */
static int scan_window(const orc_fd_scene* sc, const uint8_t* lbp, int W, int x, int y, uint64_t* survivors) {
  const int32_t* wk = sc->weak;
  for (int k = 0; k < sc->n_stages; ++k) {
    int32_t s = 0;
    for (int w = 0; w < sc->n_weak[k]; ++w, wk += 12) {
      uint8_t code = lbp[(size_t)(y + wk[1]) * W + x + wk[0]];
      uint32_t bit = ((uint32_t)wk[2 + (code >> 5)] >> (code & 31)) & 1u;
      s += bit ? wk[10] : wk[11];
    }
    if (s < sc->thr[k]) return 0;
    survivors[k]++;
  }
  return 1;
}

static void fd_out_reset(const orc_fd_scene* sc, orc_fd_out* out) {
  memset(out->survivors, 0, sizeof(out->survivors));
  out->n_det = 0;
  out->windows = 0;
  memset(out->deq, 0, sizeof(out->deq));
  memset(out->hist, 0, sizeof(uint32_t) * 256 * (size_t)sc->n_frames);
  out->trace_n = 0;
}

static void add_det(orc_fd_out* out, int f, int l, int x, int y) {
  if (out->n_det < out->det_cap) {
    out->det[4 * out->n_det + 0] = (uint32_t)f;
    out->det[4 * out->n_det + 1] = (uint32_t)l;
    out->det[4 * out->n_det + 2] = (uint32_t)x;
    out->det[4 * out->n_det + 3] = (uint32_t)y;
  }
  out->n_det++;
}

/* ---------- definition oracle: direct loops ---------- */
int orc_fd_definition(const orc_fd_scene* sc, orc_fd_out* out) {
  fd_out_reset(sc, out);
  int Ws[8], Hs[8];
  const int L = orc_fd_levels(sc->W, sc->H, Ws, Hs);
  const size_t per = lvl_off(Ws, Hs, L), npx = (size_t)sc->W * sc->H;
  for (int f = 0; f < sc->n_frames; ++f) {
    const uint8_t* rgb = sc->rgb + (size_t)f * npx * 3;
    uint8_t* img = out->levels + (size_t)f * per;
    uint8_t* lbp = out->lbp + (size_t)f * per;
    uint32_t* hist = out->hist + 256 * (size_t)f;
    uint8_t* lut = out->lut + 256 * (size_t)f;
    for (size_t p = 0; p < npx; ++p) hist[fd_gray(rgb + 3 * p)]++;
    orc_histeq_lut(hist, npx, lut);
    for (size_t p = 0; p < npx; ++p) img[p] = lut[fd_gray(rgb + 3 * p)];
    for (int l = 1; l < L; ++l) {
      const uint8_t* src = img + lvl_off(Ws, Hs, l - 1);
      uint8_t* dst = img + lvl_off(Ws, Hs, l);
      for (int y = 0; y < Hs[l]; ++y)
        for (int x = 0; x < Ws[l]; ++x) dst[(size_t)y * Ws[l] + x] = src[(size_t)((5 * y) >> 2) * Ws[l - 1] + ((5 * x) >> 2)];
    }
    for (int l = 0; l < L; ++l) {
      const uint8_t* im = img + lvl_off(Ws, Hs, l);
      uint8_t* lb = lbp + lvl_off(Ws, Hs, l);
      for (int y = 0; y < Hs[l]; ++y)
        for (int x = 0; x < Ws[l]; ++x) lb[(size_t)y * Ws[l] + x] = lbp_at(im, Ws[l], Hs[l], x, y);
      for (int y = 0; y + WIN <= Hs[l]; ++y)
        for (int x = 0; x + WIN <= Ws[l]; ++x) {
          out->windows++;
          if (scan_window(sc, lb, Ws[l], x, y, out->survivors)) add_det(out, f, l, x, y);
        }
    }
  }
  return 0;
}

/* ---------- pipeline oracle ---------- */
/* stages: 0 Gray(band) 1 CDF(frame) 2 Map(band) 3 Resize(level, band) 4 LBP(level, band)
 *         5 Scan(level, window row)                                               */
typedef struct fd_item { uint32_t frame, level, a, pad; } fd_item; /* a = band or row */

typedef struct fd_user {
  const orc_fd_scene* sc;
  orc_fd_out* out;
  int L, Ws[8], Hs[8], nb[8];
  size_t per;
  int32_t* lat;      /* per frame: [cdf][resize l,b][lbp l,b][scan l,g] */
  size_t lat_per, off_rs[8], off_lbp[8], off_scan[8];
} fd_user;

static int nbands(int h) { return (h + BAND - 1) / BAND; }

/* source bands of level l-1 read by band b of level l: rows (5y)>>2 for y in the band */
static void resize_src(const fd_user* u, int l, int b, int* b0, int* b1) {
  int y0 = b * BAND, y1 = y0 + BAND - 1;
  if (y1 > u->Hs[l] - 1) y1 = u->Hs[l] - 1;
  *b0 = ((5 * y0) >> 2) / BAND;
  *b1 = ((5 * y1) >> 2) / BAND;
}

static int32_t* L_rs(fd_user* u, uint32_t f, int l, int b) { return &u->lat[f * u->lat_per + u->off_rs[l] + b]; }
static int32_t* L_lbp(fd_user* u, uint32_t f, int l, int b) { return &u->lat[f * u->lat_per + u->off_lbp[l] + b]; }
static int32_t* L_scan(fd_user* u, uint32_t f, int l, int g) { return &u->lat[f * u->lat_per + u->off_scan[l] + g]; }

/* image band (l, b) complete: arrive on LBP (l, b-1..b+1) and Resize (l+1, b') latches */
static void image_band_done(orc_engine* e, fd_user* u, uint32_t f, int l, int b) {
  for (int d = -1; d <= 1; ++d) {
    int bb = b + d;
    if (bb < 0 || bb >= u->nb[l]) continue;
    if (--*L_lbp(u, f, l, bb) == 0) {
      fd_item it = {f, (uint32_t)l, (uint32_t)bb, 0};
      orc_push(e, 4, &it);
    }
  }
  if (l + 1 < u->L)
    for (int bb = 0; bb < u->nb[l + 1]; ++bb) {
      int s0, s1;
      resize_src(u, l + 1, bb, &s0, &s1);
      if (b < s0 || b > s1) continue;
      if (--*L_rs(u, f, l + 1, bb) == 0) {
        fd_item it = {f, (uint32_t)(l + 1), (uint32_t)bb, 0};
        orc_push(e, 3, &it);
      }
    }
}

static void fd_exec(orc_engine* e, int stage, const void* item) {
  fd_user* u = (fd_user*)e->user;
  const orc_fd_scene* sc = u->sc;
  fd_item it;
  memcpy(&it, item, sizeof(it));
  orc_record(e, stage, ((uint64_t)it.frame << 40) | ((uint64_t)it.level << 32) | it.a);
  const size_t npx = (size_t)sc->W * sc->H;
  uint8_t* img = u->out->levels + (size_t)it.frame * u->per;
  uint8_t* lbp = u->out->lbp + (size_t)it.frame * u->per;
  const int l = (int)it.level;
  if (stage == 0) { /* Gray band: histogram only (level 0 is written by Map) */
    const uint8_t* rgb = sc->rgb + (size_t)it.frame * npx * 3;
    uint32_t* hist = u->out->hist + 256 * (size_t)it.frame;
    int y1 = (int)(it.a + 1) * BAND < sc->H ? (int)(it.a + 1) * BAND : sc->H;
    for (int y = (int)it.a * BAND; y < y1; ++y)
      for (int x = 0; x < sc->W; ++x) hist[fd_gray(rgb + 3 * ((size_t)y * sc->W + x))]++;
    if (--u->lat[it.frame * u->lat_per] == 0) {
      fd_item c = {it.frame, 0, 0, 0};
      orc_push(e, 1, &c);
    }
  } else if (stage == 1) { /* CDF */
    orc_histeq_lut(u->out->hist + 256 * (size_t)it.frame, npx, u->out->lut + 256 * (size_t)it.frame);
    for (int b = 0; b < u->nb[0]; ++b) {
      fd_item m = {it.frame, 0, (uint32_t)b, 0};
      orc_push(e, 2, &m);
    }
  } else if (stage == 2) { /* Map: level-0 band = LUT[gray] */
    const uint8_t* rgb = sc->rgb + (size_t)it.frame * npx * 3;
    const uint8_t* lut = u->out->lut + 256 * (size_t)it.frame;
    int y1 = (int)(it.a + 1) * BAND < sc->H ? (int)(it.a + 1) * BAND : sc->H;
    for (int y = (int)it.a * BAND; y < y1; ++y)
      for (int x = 0; x < sc->W; ++x) {
        size_t p = (size_t)y * sc->W + x;
        img[p] = lut[fd_gray(rgb + 3 * p)];
      }
    image_band_done(e, u, it.frame, 0, (int)it.a);
  } else if (stage == 3) { /* Resize band of level l */
    const uint8_t* src = img + lvl_off(u->Ws, u->Hs, l - 1);
    uint8_t* dst = img + lvl_off(u->Ws, u->Hs, l);
    int y1 = (int)(it.a + 1) * BAND < u->Hs[l] ? (int)(it.a + 1) * BAND : u->Hs[l];
    for (int y = (int)it.a * BAND; y < y1; ++y)
      for (int x = 0; x < u->Ws[l]; ++x)
        dst[(size_t)y * u->Ws[l] + x] = src[(size_t)((5 * y) >> 2) * u->Ws[l - 1] + ((5 * x) >> 2)];
    image_band_done(e, u, it.frame, l, (int)it.a);
  } else if (stage == 4) { /* LBP band of level l */
    const uint8_t* im = img + lvl_off(u->Ws, u->Hs, l);
    uint8_t* lb = lbp + lvl_off(u->Ws, u->Hs, l);
    int y1 = (int)(it.a + 1) * BAND < u->Hs[l] ? (int)(it.a + 1) * BAND : u->Hs[l];
    for (int y = (int)it.a * BAND; y < y1; ++y)
      for (int x = 0; x < u->Ws[l]; ++x) lb[(size_t)y * u->Ws[l] + x] = lbp_at(im, u->Ws[l], u->Hs[l], x, y);
    /* window-row group g needs LBP bands g and g+1 */
    for (int g = (int)it.a - 1; g <= (int)it.a; ++g) {
      if (g < 0 || g * BAND > u->Hs[l] - WIN) continue;
      if (--*L_scan(u, it.frame, l, g) == 0) {
        int ylast = g * BAND + BAND - 1 < u->Hs[l] - WIN ? g * BAND + BAND - 1 : u->Hs[l] - WIN;
        for (int y = g * BAND; y <= ylast; ++y) {
          fd_item s = {it.frame, (uint32_t)l, (uint32_t)y, 0};
          orc_push(e, 5, &s);
        }
      }
    }
  } else { /* Scan a row of windows */
    const uint8_t* lb = lbp + lvl_off(u->Ws, u->Hs, l);
    for (int x = 0; x + WIN <= u->Ws[l]; ++x) {
      u->out->windows++;
      if (scan_window(sc, lb, u->Ws[l], x, (int)it.a, u->out->survivors)) add_det(u->out, (int)it.frame, l, x, (int)it.a);
    }
  }
}

int orc_fd_pipeline(const orc_fd_scene* sc, orc_fd_out* out) {
  fd_out_reset(sc, out);
  fd_user u;
  memset(&u, 0, sizeof(u));
  u.sc = sc;
  u.out = out;
  u.L = orc_fd_levels(sc->W, sc->H, u.Ws, u.Hs);
  u.per = lvl_off(u.Ws, u.Hs, u.L);
  size_t n = 1;
  for (int l = 0; l < u.L; ++l) {
    u.nb[l] = nbands(u.Hs[l]);
    u.off_rs[l] = n;
    n += (size_t)u.nb[l];
  }
  for (int l = 0; l < u.L; ++l) {
    u.off_lbp[l] = n;
    n += (size_t)u.nb[l];
  }
  for (int l = 0; l < u.L; ++l) {
    u.off_scan[l] = n;
    n += (size_t)u.nb[l];
  }
  u.lat_per = n;
  u.lat = (int32_t*)calloc(n * (size_t)sc->n_frames, sizeof(int32_t));
  if (!u.lat) return 1;
  for (int f = 0; f < sc->n_frames; ++f) {
    int32_t* L = u.lat + (size_t)f * n;
    L[0] = u.nb[0];
    for (int l = 1; l < u.L; ++l)
      for (int b = 0; b < u.nb[l]; ++b) {
        int s0, s1;
        resize_src(&u, l, b, &s0, &s1);
        L[u.off_rs[l] + b] = s1 - s0 + 1;
      }
    for (int l = 0; l < u.L; ++l)
      for (int b = 0; b < u.nb[l]; ++b) {
        L[u.off_lbp[l] + b] = (b > 0) + 1 + (b + 1 < u.nb[l]);
        L[u.off_scan[l] + b] = 1 + (b + 1 < u.nb[l]);
      }
  }
  size_t strides[6] = {16, 16, 16, 16, 16, 16};
  orc_engine e;
  orc_engine_init(&e, 6, strides, fd_exec, &u);
  e.trace = out->trace;
  e.trace_cap = out->trace_cap;
  for (int f = 0; f < sc->n_frames; ++f)
    for (int b = 0; b < u.nb[0]; ++b) {
      fd_item it = {(uint32_t)f, 0, (uint32_t)b, 0};
      orc_push(&e, 0, &it);
    }
  int rc = orc_run(&e);
  for (int s = 0; s < 6; ++s) out->deq[s] = e.deq[s];
  out->trace_n = e.trace_n;
  orc_engine_free(&e);
  free(u.lat);
  return rc;
}

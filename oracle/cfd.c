/* cfd.c — CPU ORACLE (test infrastructure only): the CFD solver pipeline.
 *
 * PAPER.md L55 (Fig. 15: Step Factor -> Flux -> Time Step; "inner loop 3, outer loop
 * 2000"), L59, Table 1 L43 (loop, static), L37 (composite data items: "combining 1024
 * elements into one composite data item yields much better performance"), Rodinia
 * euler3d [8].  The per-cell arithmetic follows Rodinia's euler3d with
 * the readings of DESIGN.md §2 (R-F1..R-F6): a structured G x G grid, neighbours
 * (-x, +x, -y, +y), off-grid faces are far field (-2); the far-field flux contribution is
 * computed from the far-field conserved state exactly like a cell's (R-F3).
 *
 * Outer iteration: Copy (old <- vars); StepFactor; 3 x [Flux; TimeStep].
 * Definition oracle = Rodinia-order whole-grid sweeps.  Pipeline oracle = the fixpoint
 * engine over tile items (T cells of a row) with one dependency latch per (tile, parity
 * of the global RK step) and ping-pong variable buffers (R-F5).
 */
#include <math.h>
#include <stdlib.h>
#include <string.h>

#include "oracle.h"

#define GAMMA 1.4f
#define SMOOTH 0.2f
#define RKS 3
#define NV 5 /* density, momentum x/y/z, density energy */

typedef struct cell { float d, mx, my, mz, e; } cell;

static void flux_contribution(const cell* c, float vx, float vy, float vz, float p, float fmx[3], float fmy[3],
                              float fmz[3], float fe[3]) {
  fmx[0] = vx * c->mx + p;
  fmx[1] = vx * c->my;
  fmx[2] = vx * c->mz;
  fmy[0] = fmx[1];
  fmy[1] = vy * c->my + p;
  fmy[2] = vy * c->mz;
  fmz[0] = fmx[2];
  fmz[1] = fmy[2];
  fmz[2] = vz * c->mz + p;
  float de_p = c->e + p;
  fe[0] = vx * de_p;
  fe[1] = vy * de_p;
  fe[2] = vz * de_p;
}

typedef struct prim {
  float vx, vy, vz, sq, speed, p, c;
  float fmx[3], fmy[3], fmz[3], fe[3];
} prim;

static void primitives(const cell* c, prim* q) {
  q->vx = c->mx / c->d;
  q->vy = c->my / c->d;
  q->vz = c->mz / c->d;
  float sq = q->vx * q->vx + q->vy * q->vy;
  q->sq = sq + q->vz * q->vz;
  q->speed = sqrtf(q->sq);
  q->p = (GAMMA - 1.0f) * (c->e - 0.5f * c->d * q->sq);
  q->c = sqrtf(GAMMA * q->p / c->d);
  flux_contribution(c, q->vx, q->vy, q->vz, q->p, q->fmx, q->fmy, q->fmz, q->fe);
}

static cell load(const float* v, size_t n, size_t i) {
  cell c = {v[i], v[n + i], v[2 * n + i], v[3 * n + i], v[4 * n + i]};
  return c;
}

float orc_cfd_step_factor_cell(const float* vars, size_t n, size_t i, float area) {
  cell c = load(vars, n, i);
  prim q;
  primitives(&c, &q);
  return 0.5f / (sqrtf(area) * (sqrtf(q.sq) + q.c));
}

/* Rodinia compute_flux for one cell (fluxes out[5]) */
void orc_cfd_flux_cell(const orc_cfd_scene* sc, const float* vars, size_t i, float out[5]) {
  const size_t n = (size_t)sc->G * sc->G;
  cell ci = load(vars, n, i);
  prim qi;
  primitives(&ci, &qi);
  cell ff = {sc->ff[0], sc->ff[1], sc->ff[2], sc->ff[3], sc->ff[4]};
  prim qf;
  primitives(&ff, &qf);
  float fd = 0.0f, fe = 0.0f, fx = 0.0f, fy = 0.0f, fz = 0.0f;
  for (int j = 0; j < 4; ++j) {
    int nb = sc->nb[(size_t)j * n + i];
    float nx = sc->normals[((size_t)j * 3 + 0) * n + i];
    float ny = sc->normals[((size_t)j * 3 + 1) * n + i];
    float nz = sc->normals[((size_t)j * 3 + 2) * n + i];
    float nlen = nx * nx + ny * ny;
    nlen = sqrtf(nlen + nz * nz);
    if (nb >= 0) {
      cell cn = load(vars, n, (size_t)nb);
      prim qn;
      primitives(&cn, &qn);
      float factor = -nlen * SMOOTH * 0.5f * (qi.speed + sqrtf(qn.sq) + qi.c + qn.c);
      fd += factor * (ci.d - cn.d);
      fe += factor * (ci.e - cn.e);
      fx += factor * (ci.mx - cn.mx);
      fy += factor * (ci.my - cn.my);
      fz += factor * (ci.mz - cn.mz);
      float nn[3] = {nx, ny, nz};
      float mn[3] = {cn.mx, cn.my, cn.mz}, mi[3] = {ci.mx, ci.my, ci.mz};
      for (int a = 0; a < 3; ++a) {
        factor = 0.5f * nn[a];
        fd += factor * (mn[a] + mi[a]);
        fe += factor * (qn.fe[a] + qi.fe[a]);
        fx += factor * (qn.fmx[a] + qi.fmx[a]);
        fy += factor * (qn.fmy[a] + qi.fmy[a]);
        fz += factor * (qn.fmz[a] + qi.fmz[a]);
      }
    } else if (nb == -1) { /* wall */
      fx += nx * qi.p;
      fy += ny * qi.p;
      fz += nz * qi.p;
    } else if (nb == -2) { /* far field */
      float nn[3] = {nx, ny, nz};
      float mf[3] = {ff.mx, ff.my, ff.mz}, mi[3] = {ci.mx, ci.my, ci.mz};
      for (int a = 0; a < 3; ++a) {
        float factor = 0.5f * nn[a];
        fd += factor * (mf[a] + mi[a]);
        fe += factor * (qf.fe[a] + qi.fe[a]);
        fx += factor * (qf.fmx[a] + qi.fmx[a]);
        fy += factor * (qf.fmy[a] + qi.fmy[a]);
        fz += factor * (qf.fmz[a] + qi.fmz[a]);
      }
    }
  }
  out[0] = fd;
  out[1] = fx;
  out[2] = fy;
  out[3] = fz;
  out[4] = fe;
}

/* ---------- definition oracle: Rodinia-order sweeps ---------- */
int orc_cfd_definition(const orc_cfd_scene* sc, orc_cfd_out* out) {
  const size_t n = (size_t)sc->G * sc->G;
  float* vars = out->vars;
  memcpy(vars, sc->vars0, sizeof(float) * NV * n);
  float* old = (float*)malloc(sizeof(float) * NV * n);
  float* sf = (float*)malloc(sizeof(float) * n);
  float* fl = (float*)malloc(sizeof(float) * NV * n);
  if (!old || !sf || !fl) return 1;
  for (int it = 0; it < sc->n_outer; ++it) {
    memcpy(old, vars, sizeof(float) * NV * n);
    for (size_t i = 0; i < n; ++i) sf[i] = orc_cfd_step_factor_cell(vars, n, i, sc->area[i]);
    for (int j = 0; j < RKS; ++j) {
      for (size_t i = 0; i < n; ++i) {
        float f[5];
        orc_cfd_flux_cell(sc, vars, i, f);
        for (int v = 0; v < NV; ++v) fl[(size_t)v * n + i] = f[v];
      }
      for (size_t i = 0; i < n; ++i) {
        float factor = sf[i] / (float)(RKS + 1 - j);
        for (int v = 0; v < NV; ++v) vars[(size_t)v * n + i] = old[(size_t)v * n + i] + factor * fl[(size_t)v * n + i];
      }
    }
  }
  out->n_copy = out->n_step = (uint64_t)sc->n_outer * (n / (size_t)sc->T);
  out->n_flux = out->n_time = 3 * out->n_copy;
  free(old);
  free(sf);
  free(fl);
  return 0;
}

/* ---------- pipeline oracle: Copy(0) / StepFactor(1) / Flux(2) / TimeStep(3) ---------- */
typedef struct cfd_item { uint32_t tile, k, pad0, pad1; } cfd_item;

typedef struct cfd_user {
  const orc_cfd_scene* sc;
  size_t n, ntiles;
  int tpr; /* tiles per row */
  float* buf[2];
  float* old;
  float* sf;
  float* fl;
  int32_t* latch[2];
} cfd_user;

static int tile_neighbours(const cfd_user* u, uint32_t t, uint32_t nbt[4]) {
  int r = (int)t / u->tpr, q = (int)t % u->tpr, G = u->sc->G, m = 0;
  if (q > 0) nbt[m++] = t - 1;
  if (q < u->tpr - 1) nbt[m++] = t + 1;
  if (r > 0) nbt[m++] = t - (uint32_t)u->tpr;
  if (r < G - 1) nbt[m++] = t + (uint32_t)u->tpr;
  return m;
}

static void flux_arrive(orc_engine* e, cfd_user* u, uint32_t t, uint32_t k) {
  int32_t* lat = &u->latch[k & 1][t];
  if (--*lat == 0) {
    uint32_t nbt[4];
    *lat = tile_neighbours(u, t, nbt) + 1; /* re-arm for k + 2 before releasing Flux(k) */
    cfd_item f = {t, k, 0, 0};
    orc_push(e, 2, &f);
  }
}

static void cfd_exec(orc_engine* e, int stage, const void* item) {
  cfd_user* u = (cfd_user*)e->user;
  const orc_cfd_scene* sc = u->sc;
  cfd_item it;
  memcpy(&it, item, sizeof(it));
  orc_record(e, stage, ((uint64_t)it.k << 32) | it.tile);
  const size_t n = u->n, T = (size_t)sc->T, i0 = (size_t)it.tile * T;
  const uint32_t k = it.k;
  float* cur = u->buf[k & 1];
  if (stage == 0) { /* Copy: old <- vars (the state at global RK step k = 3 * outer) */
    for (int v = 0; v < NV; ++v) memcpy(u->old + (size_t)v * n + i0, cur + (size_t)v * n + i0, sizeof(float) * T);
    orc_push(e, 1, &it);
  } else if (stage == 1) { /* StepFactor */
    for (size_t i = i0; i < i0 + T; ++i) u->sf[i] = orc_cfd_step_factor_cell(cur, n, i, sc->area[i]);
    flux_arrive(e, u, it.tile, k);
  } else if (stage == 2) { /* Flux */
    for (size_t i = i0; i < i0 + T; ++i) {
      float f[5];
      orc_cfd_flux_cell(sc, cur, i, f);
      for (int v = 0; v < NV; ++v) u->fl[(size_t)v * n + i] = f[v];
    }
    orc_push(e, 3, &it);
  } else { /* TimeStep: vars(k+1) = old + sf / (RK + 1 - rk) * flux */
    const int rk = (int)(k % RKS);
    const uint32_t outer = k / RKS;
    float* nxt = u->buf[(k + 1) & 1];
    for (size_t i = i0; i < i0 + T; ++i) {
      float factor = u->sf[i] / (float)(RKS + 1 - rk);
      for (int v = 0; v < NV; ++v) nxt[(size_t)v * n + i] = u->old[(size_t)v * n + i] + factor * u->fl[(size_t)v * n + i];
    }
    if (outer + (rk == RKS - 1 ? 1u : 0u) >= (uint32_t)sc->n_outer) return; /* last step */
    uint32_t nbt[4];
    int m = tile_neighbours(u, it.tile, nbt);
    for (int j = 0; j < m; ++j) flux_arrive(e, u, nbt[j], k + 1);
    if (rk < RKS - 1) {
      flux_arrive(e, u, it.tile, k + 1);
    } else {
      cfd_item c = {it.tile, k + 1, 0, 0};
      orc_push(e, 0, &c);
    }
  }
}

int orc_cfd_pipeline(const orc_cfd_scene* sc, orc_cfd_out* out) {
  cfd_user u;
  memset(&u, 0, sizeof(u));
  u.sc = sc;
  u.n = (size_t)sc->G * sc->G;
  u.ntiles = u.n / (size_t)sc->T;
  u.tpr = sc->G / sc->T;
  if (sc->T > sc->G || sc->G % sc->T) return 1;
  u.buf[0] = (float*)malloc(sizeof(float) * NV * u.n);
  u.buf[1] = (float*)malloc(sizeof(float) * NV * u.n);
  u.old = (float*)malloc(sizeof(float) * NV * u.n);
  u.sf = (float*)malloc(sizeof(float) * u.n);
  u.fl = (float*)malloc(sizeof(float) * NV * u.n);
  u.latch[0] = (int32_t*)malloc(sizeof(int32_t) * u.ntiles);
  u.latch[1] = (int32_t*)malloc(sizeof(int32_t) * u.ntiles);
  if (!u.buf[0] || !u.buf[1] || !u.old || !u.sf || !u.fl || !u.latch[0] || !u.latch[1]) return 1;
  memcpy(u.buf[0], sc->vars0, sizeof(float) * NV * u.n);
  for (size_t t = 0; t < u.ntiles; ++t) {
    uint32_t nbt[4];
    u.latch[0][t] = 1; /* k = 0: initial values are final, only the tile's StepFactor arrives */
    u.latch[1][t] = tile_neighbours(&u, (uint32_t)t, nbt) + 1;
  }
  size_t strides[4] = {16, 16, 16, 16};
  orc_engine e;
  orc_engine_init(&e, 4, strides, cfd_exec, &u);
  e.trace = out->trace;
  e.trace_cap = out->trace_cap;
  if (sc->n_outer > 0)
    for (size_t t = 0; t < u.ntiles; ++t) {
      cfd_item c = {(uint32_t)t, 0, 0, 0};
      orc_push(&e, 0, &c);
    }
  int rc = orc_run(&e);
  out->n_copy = e.deq[0];
  out->n_step = e.deq[1];
  out->n_flux = e.deq[2];
  out->n_time = e.deq[3];
  out->trace_n = e.trace_n;
  memcpy(out->vars, u.buf[(3 * (size_t)sc->n_outer) & 1], sizeof(float) * NV * u.n);
  orc_engine_free(&e);
  free(u.buf[0]);
  free(u.buf[1]);
  free(u.old);
  free(u.sf);
  free(u.fl);
  free(u.latch[0]);
  free(u.latch[1]);
  return rc;
}

/* ldpc.c — CPU ORACLE (test infrastructure only): the LDPC decoder pipeline of PAPER.md
 * Fig. 17 (L59: "LDPC (Low-Density Parity-Check) [15] is a linear error correction
 * program ... There are 4 stages in LDPC decoding pipeline" -- Initialize, C2V, V2C,
 * ProbVar, with an inner loop; L53 "we set both the number of frames and iterations as
 * 100"; Table 1: Loop / Static; Table 2: 12-B items).
 *
 * The paper gives no decoding arithmetic (its code is from [18]).  DESIGN.md readings
 * R-L1..R-L6: normalised min-sum message passing on a (3,6)-regular parity-check matrix
 * H given as data (edges in check-major order), float32, fixed summation order:
 *   Initialize(f):      v2c[e] = L[var(e)]
 *   C2V(f, it):         c2v[e] = s_e * (alpha * min_{e' in chk(e), e' != e} |v2c[e']|),
 *                       s_e = prod_{e' != e} sgn(v2c[e']), sgn(x) = x < 0 ? -1 : +1
 *   V2C(f, it):         v2c[e] = L[n] + sum_{e' in var(n), e' != e} c2v[e'] (edge order)
 *   ProbVar(f, it):     P[n] = L[n] + sum_{e in var(n)} c2v[e] (edge order);
 *                       bit[n] = P[n] < 0; errors[f][it] = #(bit != 0) (all-zero codeword);
 *                       it + 1 < iters ? C2V(f, it + 1) : output P
 * Two layers: a definition (plain per-frame loops) and the pipeline through fixpoint.c.
 */
#include <math.h>
#include <stdlib.h>
#include <string.h>

#include "oracle.h"

static float sgn_mag(int neg, float mag) { return neg ? -mag : mag; }

/* Check node m: edges [m*dc, (m+1)*dc). */
static void c2v_check(const orc_ldpc* d, const float* v2c, float* c2v, int m) {
  for (int k = 0; k < d->dc; ++k) {
    const int e = m * d->dc + k;
    float mag = INFINITY;
    int neg = 0;
    for (int j = 0; j < d->dc; ++j) {
      if (j == k) continue;
      const float x = v2c[m * d->dc + j];
      const float a = fabsf(x);
      if (a < mag) mag = a;
      neg ^= x < 0.0f;
    }
    c2v[e] = sgn_mag(neg, d->alpha * mag);
  }
}

/* Variable node n: edges var_edges[n*dv .. n*dv+dv). */
static void v2c_var(const orc_ldpc* d, const float* L, const float* c2v, float* v2c, int n) {
  for (int k = 0; k < d->dv; ++k) {
    float acc = L[n];
    for (int j = 0; j < d->dv; ++j) {
      if (j == k) continue;
      acc = acc + c2v[d->var_edges[n * d->dv + j]];
    }
    v2c[d->var_edges[n * d->dv + k]] = acc;
  }
}

static float posterior(const orc_ldpc* d, const float* L, const float* c2v, int n) {
  float acc = L[n];
  for (int j = 0; j < d->dv; ++j) acc = acc + c2v[d->var_edges[n * d->dv + j]];
  return acc;
}

static int check_desc(const orc_ldpc* d) {
  if (d->N <= 0 || d->M <= 0 || d->dv <= 0 || d->dc <= 1 || d->N * d->dv != d->M * d->dc) return 1;
  if (d->n_frames <= 0 || d->n_iter <= 0) return 1;
  return 0;
}

/* Definition: per frame, the textbook decoding loop. */
int orc_ldpc_definition(const orc_ldpc* d, float* post, int32_t* errors) {
  if (check_desc(d)) return 1;
  const size_t E = (size_t)d->N * d->dv;
  float* v2c = (float*)malloc(E * sizeof(float));
  float* c2v = (float*)malloc(E * sizeof(float));
  if (!v2c || !c2v) { free(v2c); free(c2v); return 1; }
  for (int f = 0; f < d->n_frames; ++f) {
    const float* L = d->llr + (size_t)f * d->N;
    for (size_t e = 0; e < E; ++e) v2c[e] = L[d->check_vars[e]];
    for (int it = 0; it < d->n_iter; ++it) {
      for (int m = 0; m < d->M; ++m) c2v_check(d, v2c, c2v, m);
      for (int n = 0; n < d->N; ++n) v2c_var(d, L, c2v, v2c, n);
      int err = 0;
      for (int n = 0; n < d->N; ++n) {
        const float P = posterior(d, L, c2v, n);
        err += P < 0.0f;
        if (it == d->n_iter - 1) post[(size_t)f * d->N + n] = P;
      }
      errors[(size_t)f * d->n_iter + it] = err;
    }
  }
  free(v2c);
  free(c2v);
  return 0;
}

/* Pipeline (reading R-L6): items {frame, iteration, chunk}.  Initialize(f) emits the
 * nc_chk C2V chunks of iteration 0; the last C2V chunk of (f, it) to finish (a dependency
 * latch) emits the nc_var V2C and nc_var ProbVar chunks of (f, it); the last of those 2*nc_var
 * chunks emits the C2V chunks of (f, it + 1) -- ProbVar(it) must read c2v before C2V(it+1)
 * overwrites it.  Chunk c of n covers [c*K/n, (c+1)*K/n) of the K checks or variables. */
typedef struct ldpc_item { uint32_t frame, iter, chunk, pad; } ldpc_item;
typedef struct ldpc_user {
  const orc_ldpc* d;
  float *v2c, *c2v, *post;
  int32_t* errors;
  int32_t* latch_c;  /* [frames] C2V chunks of the current iteration still to finish   */
  int32_t* latch_v;  /* [frames] V2C + ProbVar chunks still to finish                  */
} ldpc_user;

static void ldpc_exec(orc_engine* eng, int stage, const void* p) {
  ldpc_user* u = (ldpc_user*)eng->user;
  const orc_ldpc* d = u->d;
  ldpc_item it;
  memcpy(&it, p, sizeof(it));
  const size_t E = (size_t)d->N * d->dv;
  float* v2c = u->v2c + (size_t)it.frame * E;
  float* c2v = u->c2v + (size_t)it.frame * E;
  const float* L = d->llr + (size_t)it.frame * d->N;
  orc_record(eng, stage, ((uint64_t)it.frame << 32) | ((uint64_t)it.iter << 8) | it.chunk);
  if (stage == 0) {          /* Initialize */
    for (size_t e = 0; e < E; ++e) v2c[e] = L[d->check_vars[e]];
    for (int c = 0; c < d->nc_chk; ++c) {
      ldpc_item x = {it.frame, 0u, (uint32_t)c, 0u};
      orc_push(eng, 1, &x);
    }
  } else if (stage == 1) {   /* C2V chunk */
    const int m0 = (int)((long long)it.chunk * d->M / d->nc_chk), m1 = (int)((long long)(it.chunk + 1) * d->M / d->nc_chk);
    for (int m = m0; m < m1; ++m) c2v_check(d, v2c, c2v, m);
    if (--u->latch_c[it.frame] == 0) {
      u->latch_c[it.frame] = d->nc_chk;
      for (int c = 0; c < d->nc_var; ++c) {
        ldpc_item x = {it.frame, it.iter, (uint32_t)c, 0u};
        orc_push(eng, 2, &x);
        orc_push(eng, 3, &x);
      }
    }
  } else {                   /* V2C / ProbVar chunk */
    const int n0 = (int)((long long)it.chunk * d->N / d->nc_var), n1 = (int)((long long)(it.chunk + 1) * d->N / d->nc_var);
    if (stage == 2) {
      for (int n = n0; n < n1; ++n) v2c_var(d, L, c2v, v2c, n);
    } else {
      int err = 0;
      for (int n = n0; n < n1; ++n) {
        const float P = posterior(d, L, c2v, n);
        err += P < 0.0f;
        if ((int)it.iter == d->n_iter - 1) u->post[(size_t)it.frame * d->N + n] = P;
      }
      u->errors[(size_t)it.frame * d->n_iter + it.iter] += err;
    }
    if (--u->latch_v[it.frame] == 0) {
      u->latch_v[it.frame] = 2 * d->nc_var;
      if ((int)it.iter + 1 < d->n_iter)
        for (int c = 0; c < d->nc_chk; ++c) {
          ldpc_item x = {it.frame, it.iter + 1u, (uint32_t)c, 0u};
          orc_push(eng, 1, &x);  /* inner loop back to C2V */
        }
    }
  }
}

int orc_ldpc_pipeline(const orc_ldpc* d, float* post, int32_t* errors, orc_stats* st) {
  if (check_desc(d) || d->nc_chk < 1 || d->nc_var < 1 || d->nc_chk > d->M || d->nc_var > d->N) return 1;
  const size_t E = (size_t)d->N * d->dv;
  ldpc_user u = {d, (float*)malloc(E * d->n_frames * sizeof(float)), (float*)malloc(E * d->n_frames * sizeof(float)),
                 post, errors, (int32_t*)malloc(sizeof(int32_t) * d->n_frames), (int32_t*)malloc(sizeof(int32_t) * d->n_frames)};
  if (!u.v2c || !u.c2v || !u.latch_c || !u.latch_v) {
    free(u.v2c); free(u.c2v); free(u.latch_c); free(u.latch_v);
    return 1;
  }
  memset(errors, 0, sizeof(int32_t) * (size_t)d->n_frames * d->n_iter);
  for (int f = 0; f < d->n_frames; ++f) {
    u.latch_c[f] = d->nc_chk;
    u.latch_v[f] = 2 * d->nc_var;
  }
  size_t strides[4] = {16, 16, 16, 16};
  orc_engine e;
  orc_engine_init(&e, 4, strides, ldpc_exec, &u);
  for (int f = 0; f < d->n_frames; ++f) {
    ldpc_item it = {(uint32_t)f, 0u, 0u, 0u};
    orc_push(&e, 0, &it);
  }
  int rc = orc_run(&e);
  if (st) {
    memset(st, 0, sizeof(*st));
    for (int s = 0; s < 4; ++s) { st->deq[s] = e.deq[s]; st->enq[s] = e.enq[s]; }
  }
  orc_engine_free(&e);
  free(u.v2c);
  free(u.c2v);
  free(u.latch_c);
  free(u.latch_v);
  return rc;
}

/* toy.c — CPU ORACLE (test infrastructure only): the Fig. 9 programming example.
 *
 * PAPER.md L37 (§6, Fig. 9): "Stage 1 ... each data item is multiplied by 2. If the
 * value reaches a threshold, the data item is enqueued for stage 2 to process;
 * otherwise, it goes through stage 1 again."  Stages 2 and 3 are elided in the paper
 * ("...; // Definition of Stage_2 and Stage_3"); reading R-T1: Stage 2 adds 1
 * and forwards to Stage 3, Stage 3 is the sink.  THRESHOLD = 2^20 (reading R-T2);
 * inputs are in [1, THRESHOLD).
 */
#include <stdlib.h>
#include <string.h>

#include "oracle.h"

/* Definition: the loop the recursive stage unrolls into. */
int orc_toy_definition(const int32_t* in, size_t n, int32_t threshold, int32_t* out, uint64_t* s1_passes) {
  uint64_t passes = 0;
  for (size_t i = 0; i < n; ++i) {
    int32_t v = in[i];
    if (v <= 0) return 1; /* never terminates: outside the generator's domain */
    do {
      v *= 2;
      passes++;
    } while (v < threshold);
    out[i] = v + 1;
  }
  if (s1_passes) *s1_passes = passes;
  return 0;
}

typedef struct toy_user {
  int32_t threshold;
  int32_t* out;
  size_t n_out;
} toy_user;

static void toy_exec(orc_engine* e, int stage, const void* item) {
  toy_user* u = (toy_user*)e->user;
  int32_t v;
  memcpy(&v, item, 4);
  if (stage == 0) { /* Stage_1::execute, Fig. 9 */
    v *= 2;
    if (v >= u->threshold) orc_push(e, 1, &v);
    else orc_push(e, 0, &v);
  } else if (stage == 1) { /* Stage_2 (reading R-T1) */
    v += 1;
    orc_push(e, 2, &v);
  } else { /* Stage_3: sink */
    u->out[u->n_out++] = v;
  }
}

int orc_toy_pipeline(const int32_t* in, size_t n, int32_t threshold, int32_t* out, size_t* n_out,
                     orc_stats* st) {
  size_t strides[3] = {4, 4, 4};
  toy_user u = {threshold, out, 0};
  orc_engine e;
  orc_engine_init(&e, 3, strides, toy_exec, &u);
  for (size_t i = 0; i < n; ++i) {
    if (in[i] <= 0) { orc_engine_free(&e); return 1; }
    orc_push(&e, 0, &in[i]); /* VersaPipe::insertIntoQueue(initItems, n) */
  }
  int rc = orc_run(&e);
  if (st) {
    memset(st, 0, sizeof(*st));
    for (int s = 0; s < 3; ++s) { st->deq[s] = e.deq[s]; st->enq[s] = e.enq[s]; }
  }
  *n_out = u.n_out;
  orc_engine_free(&e);
  return rc;
}

/* qbench.c — CPU ORACLE (test infrastructure only): the queue microbenchmark pipeline
 * (not a paper workload).
 *
 * One self-recursive stage (item of 4, 16 or 272 bytes).  Word 0 of an item is
 * id | depth << 24; a non-leaf item (fanout > 0 and depth > 0) pushes `fanout` copies of
 * itself with depth - 1 (the payload words are copied unchanged); a leaf checks that
 * payload word k equals id * 2654435761 + k * 40503 (mod 2^32) and is counted.  Run by
 * the generic sequential engine (fixpoint.c).  Closed forms (tests/test_oracle_qbench.py):
 * tasks per seed = 1 (fan-out 0), depth + 1 (fan-out 1), 2^(depth+1) - 1 (fan-out 2).
 */
#include <stdlib.h>
#include <string.h>

#include "oracle.h"

typedef struct qb_user {
  uint32_t fanout;
  size_t words;
  uint64_t leaves, idsum, bad;
} qb_user;

static void qb_exec(orc_engine* e, int stage, const void* item) {
  qb_user* u = (qb_user*)e->user;
  uint32_t w[68];
  memcpy(w, item, u->words * 4);
  uint32_t id = w[0] & 0xffffffu, d = w[0] >> 24;
  if (u->fanout == 0 || d == 0) {
    int bad = 0;
    for (size_t k = 1; k < u->words; ++k) bad |= w[k] != (uint32_t)(id * 2654435761u + (uint32_t)k * 40503u);
    u->leaves++;
    u->idsum += id;
    u->bad += (uint64_t)bad;
    return;
  }
  w[0] = id | ((d - 1) << 24);
  for (uint32_t c = 0; c < u->fanout; ++c) orc_push(e, stage, w);
}

int orc_qbench_pipeline(const void* seeds, size_t n, size_t item_bytes, uint32_t fanout, uint64_t* leaves,
                        uint64_t* idsum, uint64_t* bad, orc_stats* st) {
  if (item_bytes != 4 && item_bytes != 16 && item_bytes != 272) return 1;
  if (fanout > 2) return 1;
  size_t strides[1] = {item_bytes};
  qb_user u = {fanout, item_bytes / 4, 0, 0, 0};
  orc_engine e;
  orc_engine_init(&e, 1, strides, qb_exec, &u);
  for (size_t i = 0; i < n; ++i) orc_push(&e, 0, (const uint8_t*)seeds + i * item_bytes);
  int rc = orc_run(&e);
  if (st) {
    memset(st, 0, sizeof(*st));
    st->deq[0] = e.deq[0];
    st->enq[0] = e.enq[0];
  }
  *leaves = u.leaves;
  *idsum = u.idsum;
  *bad = u.bad;
  orc_engine_free(&e);
  return rc;
}

/* collatz.c — CPU ORACLE (test infrastructure only): the Collatz queue-stress pipeline.
 *
 * Not a paper workload (reading R-C1): a deep, irregular,
 * data-dependent recursion with 16-B items used to stress the runtime invariants of
 * SURVEY §8(c-6).  Item {u32 id, u32 steps, u64 v}.
 *   S1: if v == 1 -> sink; else v <- (v even ? v/2 : 3v+1), steps++, back to S1.
 *   S2 (sink): steps_out[id] = steps, seen[id]++.
 */
#include <string.h>

#include "oracle.h"

int orc_collatz_definition(const orc_collatz_item* in, size_t n, uint32_t* steps_out) {
  for (size_t i = 0; i < n; ++i) {
    uint64_t v = in[i].v;
    uint32_t s = in[i].steps;
    if (v == 0) return 1;
    while (v != 1) {
      v = (v % 2 == 0) ? v / 2 : 3 * v + 1;
      s++;
    }
    steps_out[in[i].id] = s;
  }
  return 0;
}

typedef struct collatz_user {
  uint32_t max_steps;
  uint32_t* steps_out;
  uint32_t* seen;
} collatz_user;

static void collatz_exec(orc_engine* e, int stage, const void* item) {
  collatz_user* u = (collatz_user*)e->user;
  orc_collatz_item it;
  memcpy(&it, item, sizeof(it));
  orc_record(e, stage, ((uint64_t)it.id << 32) | it.steps);
  if (stage == 0) {
    if (it.v == 1) {
      orc_push(e, 1, &it);
    } else {
      if (it.steps >= u->max_steps) { e->error = 2; return; } /* recursion-depth guard */
      it.v = (it.v % 2 == 0) ? it.v / 2 : 3 * it.v + 1;
      it.steps++;
      orc_push(e, 0, &it);
    }
  } else {
    u->steps_out[it.id] = it.steps;
    u->seen[it.id]++;
  }
}

int orc_collatz_pipeline(const orc_collatz_item* in, size_t n, uint32_t max_steps, uint32_t* steps_out,
                         uint32_t* seen, orc_stats* st) {
  size_t strides[2] = {sizeof(orc_collatz_item), sizeof(orc_collatz_item)};
  collatz_user u = {max_steps, steps_out, seen};
  orc_engine e;
  orc_engine_init(&e, 2, strides, collatz_exec, &u);
  for (size_t i = 0; i < n; ++i) orc_push(&e, 0, &in[i]);
  int rc = orc_run(&e);
  if (st) {
    memset(st, 0, sizeof(*st));
    for (int s = 0; s < 2; ++s) { st->deq[s] = e.deq[s]; st->enq[s] = e.enq[s]; }
  }
  orc_engine_free(&e);
  return rc;
}

"""Pins for the toy (Fig. 9) and Collatz (SURVEY c-0b) oracles.

Each check is independent of the oracle's own code: closed forms derived from the
definition, textbook values, and brute force in pure Python.
"""
import json
import os

import numpy as np

from paper_conf_micro_zhengozsyc17_b200 import inputs

GOLDEN = os.path.join(os.path.dirname(__file__), "golden")


def toy_closed_form(v: int, T: int):
    """Fig. 9 Stage_1 doubles until v >= T: k(v) = max(1, ceil(log2(T/v))) passes,
    output (Stage_2 adds 1, reading R-T1) v*2^k + 1.  ceil(log2(T/v)) over the integers:
    smallest k with 2^k >= ceil(T/v)."""
    r = -(-T // v)
    k = max(1, (r - 1).bit_length())
    return k, v * (1 << k) + 1


def test_toy_closed_form_and_counts(orc):
    T = inputs.TOY_THRESHOLD
    seeds = inputs.toy_seeds(5000)
    seeds = np.concatenate([seeds, np.array([1, 2, T - 1, T // 2, T // 2 + 1, T // 4], np.int32)])
    ks, outs = zip(*(toy_closed_form(int(v), T) for v in seeds))
    out_def, passes = orc.toy_definition(seeds, T)
    assert out_def.tolist() == list(outs)
    assert passes == sum(ks)
    out_pipe, deq, enq = orc.toy_pipeline(seeds, T)
    assert sorted(out_pipe.tolist()) == sorted(outs)
    n = len(seeds)
    assert deq == [sum(ks), n, n]
    # seeds count as enq of stage 1; every pass but the last re-enqueues to stage 1
    assert enq == [n + sum(ks) - n, n, n]


def test_toy_fig9_example(orc):
    """Fig. 9: insertIntoQueue(initItems, 10).  THRESHOLD = 2^20 (reading R-T2)."""
    T = inputs.TOY_THRESHOLD
    init = np.array([1, 3, 7, 100, 1000, 4096, 65535, 65536, 524288, 1048575], np.int32)
    out, deq, _ = orc.toy_pipeline(init, T)
    # hand-derived: 1 -> 2^20 after 20 passes (+1); 524288 = 2^19 -> 2^20 after 1 pass;
    # 1048575 = T-1 -> one pass to 2097150.
    assert sorted(out.tolist()) == sorted([toy_closed_form(int(v), T)[1] for v in init])
    assert (1 << 20) + 1 in out.tolist()
    assert 2097150 + 1 in out.tolist()
    assert deq[1] == deq[2] == 10


def collatz_py(v: int) -> int:
    s = 0
    while v != 1:
        v = v // 2 if v % 2 == 0 else 3 * v + 1
        s += 1
    return s


def test_collatz_textbook_values(orc):
    """Textbook stopping times (golden/collatz_textbook.json, with their source)."""
    g = json.load(open(os.path.join(GOLDEN, "collatz_textbook.json")))
    vals = sorted(int(k) for k in g["total_stopping_time"])
    a = np.zeros(len(vals), inputs.COLLATZ_DTYPE)
    a["id"] = np.arange(len(vals))
    a["v"] = vals
    out = orc.collatz_definition(a)
    assert [int(x) for x in out] == [g["total_stopping_time"][str(v)] for v in vals]
    rc, out2, seen, deq, enq = orc.collatz_pipeline(a)
    assert rc == 0 and np.array_equal(out, out2) and np.all(seen == 1)


def test_collatz_pipeline_conservation(orc):
    seeds = inputs.collatz_seeds(3000)
    ref = [collatz_py(int(v)) for v in seeds["v"]]
    rc, out, seen, deq, enq = orc.collatz_pipeline(seeds)
    assert rc == 0
    assert out.tolist() == ref
    assert np.all(seen == 1)                     # each id reaches the sink exactly once
    assert deq[0] == sum(ref) + len(ref)         # SURVEY c-0b: deq[S1] = sum(stopping time + 1)
    assert deq[1] == len(ref)
    assert sum(enq) == sum(deq)                  # Σ enq == Σ deq (seeds counted as enq)


def test_collatz_depth_guard(orc):
    a = np.zeros(1, inputs.COLLATZ_DTYPE)
    a["v"] = 27
    rc, *_ = orc.collatz_pipeline(a, max_steps=50)
    assert rc != 0                               # the recursion guard fires (111 > 50)

"""CPU pins of the queue-microbenchmark oracle (oracle/qbench.c): task
counts against their closed forms, leaf id sums against the arithmetic series, and a
corrupted payload is detected (so a stage that forgets to copy the payload fails)."""
import numpy as np
import pytest

import oracle
from paper_conf_micro_zhengozsyc17_b200 import inputs


@pytest.mark.parametrize("item_bytes", [4, 16, 272])
@pytest.mark.parametrize("fanout", [0, 1, 2])
@pytest.mark.parametrize("depth", [0, 1, 6])
def test_task_counts_closed_form(item_bytes, fanout, depth):
    n = 257
    leaves, idsum, bad, deq = oracle.qbench_pipeline(inputs.qbench_seeds(n, item_bytes, depth), item_bytes, fanout)
    per_task = {0: 1, 1: depth + 1, 2: 2 ** (depth + 1) - 1}[fanout]
    per_leaf = 2 ** depth if fanout == 2 else 1
    assert deq == n * per_task
    assert leaves == n * per_leaf
    assert idsum == per_leaf * n * (n - 1) // 2
    assert bad == 0


def test_corrupted_payload_detected():
    s = inputs.qbench_seeds(10, 272, 3).reshape(10, 68).copy()
    s[4, 37] ^= 1
    leaves, _, bad, _ = oracle.qbench_pipeline(s.reshape(-1), 272, 2)
    assert leaves == 80 and bad == 8          # all 2^3 leaves of seed 4


def test_ids_wrap_at_24_bits():
    s = inputs.qbench_seeds(4, 16, 0, id0=(1 << 24) - 2)
    w = s.reshape(4, 4)[:, 0]
    assert list(w & 0xFFFFFF) == [(1 << 24) - 2, (1 << 24) - 1, 0, 1]
    assert oracle.qbench_pipeline(s, 16, 1)[2] == 0

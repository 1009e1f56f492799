"""GPU parity of the queue microbenchmark through the C ABI: every item
size x fan-out x execution model against the CPU oracle (leaves, leaf id sum, payload
integrity, tasks dequeued), plus the runtime invariants of SURVEY §8(c-6)."""
import numpy as np
import pytest

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def vpm():
    import torch
    if not torch.cuda.is_available():
        pytest.skip("needs a GPU")
    from paper_conf_micro_zhengozsyc17_b200 import vp
    return vp


def model_of(vp, name):
    return {"kbk": vp.KBK, "kbk_graph": vp.KBK_GRAPH, "megakernel": vp.MEGAKERNEL, "coarse": vp.COARSE,
            "fine": vp.FINE}[name]


@pytest.mark.parametrize("item_bytes", [4, 16, 272])
@pytest.mark.parametrize("fanout,depth", [(0, 0), (1, 9), (2, 7)])
@pytest.mark.parametrize("model", ["kbk", "kbk_graph", "megakernel", "fine"])
def test_qbench_parity(vpm, orc, item_bytes, fanout, depth, model):
    from paper_conf_micro_zhengozsyc17_b200.workloads import QBenchPipeline
    vp = vpm
    n = 20_000 if item_bytes < 272 else 4_000
    qb = QBenchPipeline(n, item_bytes, fanout, depth)
    lv, ids, bad, deq = orc.qbench_pipeline(qb.seeds, item_bytes, fanout)
    assert deq == qb.tasks()
    qb.configure(model_of(vp, model))
    for _ in range(2):
        r, st = qb.run()
        assert (r["leaves"], r["idsum"], r["bad"]) == (lv, ids, 0)
        assert st["dequeued"][qb.stage] == deq
        assert st["enqueued"][qb.stage] == deq                  # seeds + children == tasks
        assert st["abort_reason"] == 0 and st["pending"] == 0
        assert st["ring_count"][qb.stage] == 0 and st["ring_head"][qb.stage] == st["ring_tail"][qb.stage]


@pytest.mark.parametrize("batch", [1, 32, 1024])
def test_qbench_batch_sizes(vpm, orc, batch):
    from paper_conf_micro_zhengozsyc17_b200.workloads import QBenchPipeline
    vp = vpm
    qb = QBenchPipeline(50_000, 16, 1, 5)
    lv, ids, _, deq = orc.qbench_pipeline(qb.seeds, 16, 1)
    qb.configure(vp.MEGAKERNEL, None, batch)
    r, st = qb.run()
    assert (r["leaves"], r["idsum"], r["bad"]) == (lv, ids, 0) and st["dequeued"][qb.stage] == deq


def test_qbench_graph_kbk_launch_count(vpm):
    """Device-driven KBK: the while loop ran, and repeated runs reuse the instantiated graph."""
    from paper_conf_micro_zhengozsyc17_b200.workloads import QBenchPipeline
    vp = vpm
    qb = QBenchPipeline(1000, 4, 1, 20)
    qb.configure(vp.KBK_GRAPH)
    r1, st1 = qb.run()
    r2, st2 = qb.run()
    assert r1 == r2 and r1["leaves"] == 1000
    # one chain level per iteration at least: >= depth + 1 iterations of the single stage
    assert st1["kbk_launches"] >= 21 and st1["kbk_launches"] == st2["kbk_launches"]


@pytest.mark.parametrize("item_bytes", [4, 16])
@pytest.mark.parametrize("fanout,depth,n", [(2, 12, 8), (1, 30, 3000), (2, 6, 500)])
def test_qbench_cluster_steal(vpm, orc, item_bytes, fanout, depth, n):
    """the cooperative megakernel as clusters of 2 CTAs that take items from
    each other's block-local queue over DSMEM (VP_FLAG_CLUSTER_STEAL): same leaves, leaf-id
    sum and payloads as the oracle, every item dequeued exactly once, on repeated runs; and
    stealing happens (a tree grown from a few seeds starts in one CTA's local queue)."""
    from paper_conf_micro_zhengozsyc17_b200.workloads import QBenchPipeline
    vp = vpm
    qb = QBenchPipeline(n, item_bytes, fanout, depth, steal=True)
    lv, ids, bad, deq = orc.qbench_pipeline(qb.seeds, item_bytes, fanout)
    qb.configure(vp.MEGAKERNEL)
    stolen = 0
    for _ in range(3):
        r, st = qb.run()
        assert (r["leaves"], r["idsum"], r["bad"]) == (lv, ids, 0)
        assert st["dequeued"][qb.stage] == deq and st["enqueued"][qb.stage] == deq
        assert st["abort_reason"] == 0 and st["pending"] == 0
        stolen += st["stolen"][qb.stage]
    if fanout == 2 and n == 8:
        assert stolen > 0
    # the flag is a run-time one: off again, nothing is stolen
    qb.p.set_flags(0)
    r, st = qb.run()
    assert (r["leaves"], r["idsum"], r["bad"]) == (lv, ids, 0) and st["stolen"][qb.stage] == 0


@pytest.mark.parametrize("model", ["kbk", "kbk_graph", "fine"])
def test_qbench_cluster_steal_kinds_other_models(vpm, orc, model):
    """The stealing kinds under the other execution models: no cluster launch, so nothing is
    stolen and the results are those of the plain kinds."""
    from paper_conf_micro_zhengozsyc17_b200.workloads import QBenchPipeline
    vp = vpm
    for item_bytes in (4, 16):
        qb = QBenchPipeline(500, item_bytes, 2, 6, steal=True)
        lv, ids, _, deq = orc.qbench_pipeline(qb.seeds, item_bytes, 2)
        qb.configure(model_of(vp, model))
        r, st = qb.run()
        assert (r["leaves"], r["idsum"], r["bad"]) == (lv, ids, 0) and st["dequeued"][qb.stage] == deq
        assert st["stolen"][qb.stage] == 0 and st["pending"] == 0

"""GPU parity: toy (Fig. 9, L37) and Collatz stress pipelines through the C ABI, every
execution model, against the CPU oracle and closed forms."""
import numpy as np
import pytest

from paper_conf_micro_zhengozsyc17_b200 import inputs

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def vpm():
    import torch
    if not torch.cuda.is_available():
        pytest.skip("needs a GPU")
    from paper_conf_micro_zhengozsyc17_b200 import vp
    return vp


def hybrid_toy(vp, nsm):
    # [S1] megakernel on the first half, [S2,S3] RTC on the second half (Fig. 7 style)
    return vp.make_binding([(0, 0, vp.GROUP_MEGA, 0, nsm // 2), (1, 2, vp.GROUP_RTC, nsm // 2, nsm)], nsm)


@pytest.mark.parametrize("model", ["kbk", "kbk_graph", "megakernel", "coarse", "fine", "hybrid", "hybrid_kbk"])
def test_toy_all_models(vpm, orc, model):
    from paper_conf_micro_zhengozsyc17_b200.workloads import ToyPipeline
    vp = vpm
    T = inputs.TOY_THRESHOLD
    seeds = inputs.toy_seeds(200_000)
    ref_out, ref_deq, _ = orc.toy_pipeline(seeds, T)
    tp = ToyPipeline(seeds, T)
    nsm, _ = vp.device_info(0)
    if model == "hybrid":
        tp.configure(vp.HYBRID, hybrid_toy(vp, nsm))
    elif model == "hybrid_kbk":
        tp.configure(vp.HYBRID, vp.make_binding([(0, 0, vp.GROUP_MEGA, 0, nsm // 2), (1, 2, vp.GROUP_KBK, nsm // 2, nsm)], nsm))
    else:
        tp.configure({"kbk": vp.KBK, "kbk_graph": vp.KBK_GRAPH, "megakernel": vp.MEGAKERNEL, "coarse": vp.COARSE, "fine": vp.FINE}[model])
    for _ in range(2):  # repeated runs reuse the rings (monotonic tickets)
        out, st = tp.run()
        assert np.array_equal(np.sort(out), np.sort(ref_out))
        assert st["dequeued"][:3] == ref_deq
        assert st["abort_reason"] == 0


def test_toy_rtc_rejected_on_recursive_pipeline(vpm):
    from paper_conf_micro_zhengozsyc17_b200.workloads import ToyPipeline
    vp = vpm
    tp = ToyPipeline(inputs.toy_seeds(10))
    with pytest.raises(vp.VPError) as e:
        tp.configure(vp.RTC)
    assert e.value.status == vp.VP_ERR_UNSUPPORTED


def test_toy_fig9_ten_items(vpm, orc):
    from paper_conf_micro_zhengozsyc17_b200.workloads import ToyPipeline
    vp = vpm
    init = np.array([1, 3, 7, 100, 1000, 4096, 65535, 65536, 524288, 1048575], np.int32)
    ref, deq, _ = orc.toy_pipeline(init, inputs.TOY_THRESHOLD)
    tp = ToyPipeline(init)
    tp.configure(vp.MEGAKERNEL)
    out, st = tp.run()
    assert sorted(out.tolist()) == sorted(ref.tolist()) and st["dequeued"][:3] == deq


@pytest.mark.parametrize("model", ["kbk", "kbk_graph", "megakernel", "coarse", "fine"])
@pytest.mark.parametrize("batch", [0, 1, 32])
def test_collatz_conservation(vpm, orc, model, batch):
    from paper_conf_micro_zhengozsyc17_b200.workloads import CollatzPipeline
    vp = vpm
    seeds = inputs.collatz_seeds(50_000)
    rc, ref, seen_ref, deq_ref, _ = orc.collatz_pipeline(seeds)
    assert rc == 0
    cp = CollatzPipeline(seeds)
    cp.configure({"kbk": vp.KBK, "kbk_graph": vp.KBK_GRAPH, "megakernel": vp.MEGAKERNEL, "coarse": vp.COARSE, "fine": vp.FINE}[model], None, batch)
    steps, seen, st = cp.run()
    assert np.array_equal(steps, ref)
    assert np.all(seen == 1)                                    # each id reaches the sink exactly once
    assert st["dequeued"][:2] == deq_ref
    assert sum(st["enqueued"][:2]) == sum(st["dequeued"][:2])   # Σ enq == Σ deq, seeds counted


def test_collatz_trace_unique(vpm, orc):
    from paper_conf_micro_zhengozsyc17_b200.workloads import CollatzPipeline
    vp = vpm
    seeds = inputs.collatz_seeds(5000)
    cp = CollatzPipeline(seeds, flags=vp.FLAG_TRACE, trace_capacity=1 << 21)
    cp.configure(vp.MEGAKERNEL)
    steps, seen, st = cp.run()
    assert st["trace_records"] == sum(st["dequeued"][:2])


def test_tiny_capacity_rejected(vpm):
    """A ring smaller than two block batches of its producers cannot make progress."""
    from paper_conf_micro_zhengozsyc17_b200.workloads import CollatzPipeline
    vp = vpm
    cp = CollatzPipeline(inputs.collatz_seeds(1000), queue_capacity=64)
    with pytest.raises(vp.VPError) as e:
        cp.configure(vp.MEGAKERNEL, None, 256)
    assert e.value.status == vp.VP_ERR_INVALID
    cp.configure(vp.MEGAKERNEL, None, 16)          # 2 x 16 <= 64: accepted and correct
    steps, seen, _ = cp.run()
    assert np.all(seen == 1)


def test_watchdog_timeout_and_recovery(vpm, orc):
    """Fault injection: a forced device-watchdog timeout aborts the run loudly (no hang),
    and the next run on the same pipeline (rings reset) is correct."""
    from paper_conf_micro_zhengozsyc17_b200.workloads import CollatzPipeline
    vp = vpm
    seeds = inputs.collatz_seeds(1 << 20)
    cp = CollatzPipeline(seeds)
    cp.configure(vp.MEGAKERNEL)
    cp.p.set_timeout_ms(0.05)
    rc, st, msg = cp.p.run_status()
    assert rc == vp.VP_ERR_TIMEOUT and st["abort_reason"] == 1, (rc, msg)
    cp.p.set_timeout_ms(30000)
    steps, seen, _ = cp.run()
    assert np.all(seen == 1)
    assert np.array_equal(steps, orc.collatz_definition(seeds))


def test_guard_abort(vpm):
    from paper_conf_micro_zhengozsyc17_b200.workloads import CollatzPipeline
    vp = vpm
    a = np.zeros(1, inputs.COLLATZ_DTYPE)
    a["v"] = 27
    cp = CollatzPipeline(a, max_steps=50)
    cp.configure(vp.MEGAKERNEL)
    rc, st, msg = cp.p.run_status()
    assert rc == vp.VP_ERR_INVALID and st["abort_reason"] == 4


def test_binding_respects_masks_and_quotas(vpm):
    """check_sm()/check_sm_blk() (Fig. 5): blocks that stayed ran only on SMs of their
    group's mask and at most `quota` per (stage, SM)."""
    from paper_conf_micro_zhengozsyc17_b200.workloads import CollatzPipeline
    vp = vpm
    nsm, _ = vp.device_info(0)
    cp = CollatzPipeline(inputs.collatz_seeds(100_000))
    b = vp.make_binding([(0, 0, vp.GROUP_FINE, 0, nsm // 2), (1, 1, vp.GROUP_FINE, nsm // 2, nsm)], nsm,
                        blocks_per_sm=[2, 1])
    cp.configure(vp.HYBRID, b)
    steps, seen, st = cp.run()
    assert np.all(seen == 1)
    for k, (lo, hi, quota) in enumerate(st["kernels"]):
        per_sm = st["blocks_on_sm"][k]
        sm_lo, sm_hi = (0, nsm // 2) if lo == 0 else (nsm // 2, nsm)
        admitted = 0
        for sm in range(nsm):
            inside = sm_lo <= sm < sm_hi
            admitted += min(per_sm[sm], quota) if inside else 0
        assert admitted + st["fallback_admits"] >= st["admitted"][k] >= 1
        assert st["admitted"][k] <= quota * (sm_hi - sm_lo) + st["fallback_admits"]


@pytest.mark.parametrize("bad", ["overlap", "quota", "noncontig"])
def test_configure_validation(vpm, bad):
    from paper_conf_micro_zhengozsyc17_b200.workloads import ToyPipeline
    vp = vpm
    nsm, _ = vp.device_info(0)
    tp = ToyPipeline(inputs.toy_seeds(10))
    if bad == "overlap":
        b = vp.make_binding([(0, 0, vp.GROUP_MEGA, 0, 80), (1, 2, vp.GROUP_RTC, 60, nsm)], nsm)
    elif bad == "quota":
        b = vp.make_binding([(0, 2, vp.GROUP_FINE, 0, nsm)], nsm, blocks_per_sm=[64, 64, 64])
    else:
        b = vp.make_binding([(0, 0, vp.GROUP_MEGA, 0, 70), (1, 2, vp.GROUP_MEGA, 70, nsm)], nsm)
        b.group_of_stage[2] = 0
    with pytest.raises(vp.VPError) as e:
        tp.configure(vp.HYBRID, b)
    assert e.value.status == vp.VP_ERR_INVALID


def test_kbk_stage_wave_times(vpm, orc):
    """Host-driven KBK reports each stage's summed wave time (Table 2's longest-stage
    analog); stages that ran have > 0, the others 0, and their sum fits in the run."""
    from paper_conf_micro_zhengozsyc17_b200.workloads import ToyPipeline
    vp = vpm
    tp = ToyPipeline(inputs.toy_seeds(100_000))
    tp.configure(vp.KBK)
    _, st = tp.run()
    assert not any(st["stage_wave_ms"])          # only with VP_FLAG_TIMERS
    assert tp.p.set_flags(vp.FLAG_TIMERS) == 0
    _, st = tp.run()
    w = st["stage_wave_ms"]
    assert all(x > 0 for x in w[:3]) and all(x == 0 for x in w[3:])
    assert sum(w[:3]) <= st["device_ms"] * 1.05

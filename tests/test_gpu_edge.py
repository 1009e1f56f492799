"""GPU edge cases (tier rule ③): empty inputs under every model, a single item, ragged
batches that leave a partial last claim, and the degenerate geometry cases — each against
the oracle or the closed form."""
import numpy as np
import pytest

from paper_conf_micro_zhengozsyc17_b200 import inputs

pytestmark = pytest.mark.gpu

MODELS = ["kbk", "kbk_graph", "megakernel", "coarse", "fine"]


@pytest.fixture(scope="module")
def vpm():
    import torch
    if not torch.cuda.is_available():
        pytest.skip("needs a GPU")
    from paper_conf_micro_zhengozsyc17_b200 import vp
    return vp


def model_of(vp, m):
    return {"kbk": vp.KBK, "kbk_graph": vp.KBK_GRAPH, "megakernel": vp.MEGAKERNEL, "coarse": vp.COARSE,
            "fine": vp.FINE}[m]


@pytest.mark.parametrize("model", MODELS)
def test_empty_toy(vpm, model):
    """No seed at all: the run terminates at once, nothing is dequeued, pending is 0."""
    from paper_conf_micro_zhengozsyc17_b200.workloads import ToyPipeline
    tp = ToyPipeline(np.zeros(0, np.int32))
    tp.configure(model_of(vpm, model))
    for _ in range(2):
        out, st = tp.run()
        assert out.size == 0 and st["dequeued"][:3] == [0, 0, 0] and st["pending"] == 0 and st["abort_reason"] == 0


@pytest.mark.parametrize("model", MODELS + ["hybrid"])
def test_empty_reyes_frame_is_cleared(vpm, orc, model):
    """Zero patches: every pixel keeps the cleared key and colour 0 (reading R-R11)."""
    from paper_conf_micro_zhengozsyc17_b200.workloads import ReyesPipeline
    vp = vpm
    sc = inputs.reyes_config1()
    sc.seeds = sc.seeds[:0]
    rp = ReyesPipeline(sc)
    nsm, _ = vp.device_info(0)
    if model == "hybrid":
        rp.configure(vp.HYBRID, vp.make_binding([(0, 1, vp.GROUP_MEGA, 0, 60), (2, 3, vp.GROUP_RTC, 60, nsm)], nsm))
    else:
        rp.configure(model_of(vp, model))
    st = rp.run()
    key, _ = rp.keys()
    assert np.all(key == np.uint64(2**64 - 1)) and not rp.colours().any()
    assert st["dequeued"][:4] == [0, 0, 0, 0]


@pytest.mark.parametrize("n", [1, 2, 255, 257, 1023])
@pytest.mark.parametrize("model", ["megakernel", "kbk_graph"])
def test_toy_ragged_counts(vpm, orc, n, model):
    """Seed counts around the batch size (256): partial last claims, single items."""
    from paper_conf_micro_zhengozsyc17_b200.workloads import ToyPipeline
    seeds = inputs.toy_seeds(n)
    ref, deq, _ = orc.toy_pipeline(seeds, inputs.TOY_THRESHOLD)
    tp = ToyPipeline(seeds)
    tp.configure(model_of(vpm, model))
    out, st = tp.run()
    assert np.array_equal(np.sort(out), np.sort(ref)) and st["dequeued"][:3] == deq


def test_single_reyes_patch(vpm, orc):
    from paper_conf_micro_zhengozsyc17_b200.workloads import ReyesPipeline
    from test_gpu_reyes import check_against_oracle
    sc = inputs.reyes_config1()
    sc.seeds = sc.seeds[5:6].copy()
    rp = ReyesPipeline(sc)
    rp.configure(vpm.MEGAKERNEL)
    check_against_oracle(orc, sc, rp, rp.run())


def test_raster_all_degenerate(vpm, orc):
    """Every triangle has zero area: Clip culls all of them, the frame stays empty."""
    from paper_conf_micro_zhengozsyc17_b200.workloads import RasterPipeline
    sc = inputs.raster_scene(n=5000, W=320, H=180)
    sc.pos[:, 1] = sc.pos[:, 0]
    sc.pos[:, 2] = sc.pos[:, 0]
    ref = orc.raster_definition(sc)
    rp = RasterPipeline(sc)
    rp.configure(vpm.MEGAKERNEL)
    st = rp.run()
    assert np.array_equal(rp.keys(), ref["key"]) and np.all(ref["key"] == np.uint64(2**64 - 1))
    assert st["dequeued"][2] == 0 and st["dequeued"][3] == 0


@pytest.mark.parametrize("n_frames", [1, 3])
def test_ldpc_single_iteration_and_few_frames(vpm, orc, n_frames):
    from paper_conf_micro_zhengozsyc17_b200.workloads import LdpcPipeline
    sc = inputs.ldpc_scene(n_frames=n_frames, n_iter=1, N=256)
    lp = LdpcPipeline(sc)
    lp.configure(vpm.MEGAKERNEL)
    st = lp.run()
    ref = orc.ldpc_pipeline(sc)
    got = lp.results()
    assert np.array_equal(got["post"], ref["post"]) and np.array_equal(got["errors"], ref["errors"])
    assert st["dequeued"][:4] == ref["deq"]

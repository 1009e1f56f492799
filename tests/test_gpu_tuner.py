"""GPU: the offline auto-tuner (§7, Fig. 10) returns a valid
configuration that is at least as fast as both baselines it measured, and the pipeline
it configures still matches the CPU oracle bit-exactly; profiling reports occupancy."""
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


def test_autotune_reyes(vpm, orc):
    from paper_conf_micro_zhengozsyc17_b200.workloads import ReyesPipeline
    vp = vpm
    scene = inputs.reyes_config5(n_frames=32)
    rp = ReyesPipeline(scene)
    best, rep = rp.p.autotune(time_budget_s=20.0, sm_granularity=8, batch_choices=(1, 2))
    assert rep.candidates_run >= 3 and rep.best_ms > 0
    assert rep.best_ms <= min(x for x in (rep.baseline_kbk_ms, rep.baseline_mega_ms) if x > 0) + 1e-9
    assert all(rep.max_blocks_per_sm[s] >= 1 for s in range(4))
    # the tuned configuration is applied, serialisable, and correct
    s = vp.config_to_string(best)
    rp.p.configure_config(vp.config_from_string(s))
    st = rp.run()
    key, _ = rp.keys()
    for f in (0, 31):
        ref = orc.reyes_pipeline(inputs.reyes_config5(n_frames=1, frame0=f))
        assert np.array_equal(key[f], ref["key"][0])


def test_autotune_raster(vpm, orc):
    from paper_conf_micro_zhengozsyc17_b200.workloads import RasterPipeline
    scene = inputs.raster_scene(50_000, W=640, H=360)
    rp = RasterPipeline(scene)
    best, rep = rp.p.autotune(time_budget_s=15.0, sm_granularity=8)
    assert rep.best_ms > 0 and rep.candidates_run >= 3
    st = rp.run()
    ref = orc.raster_pipeline(scene)
    assert np.array_equal(rp.keys(), ref["key"])

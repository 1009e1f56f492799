"""GPU tests of the online adaptation (VP_FLAG_ONLINE):
a persistent group whose stages can receive no more items retires and the host relaunches
the next group downstream on its SMs.  Results must stay bit-exact against the oracle, the
refill grid must run only on the retired group's SMs, and the counters must balance."""
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


def sms_of(blocks_on_sm):
    return {sm for sm, n in enumerate(blocks_on_sm) if n > 0}


@pytest.mark.parametrize("split", [20, 74, 120])
def test_reyes_online_refill_parity(vpm, orc, split):
    from paper_conf_micro_zhengozsyc17_b200.workloads import ReyesPipeline
    from test_gpu_reyes import check_against_oracle
    vp = vpm
    nsm, _ = vp.device_info(0)
    scene = inputs.reyes_config5(n_frames=8, n_side=16)
    rp = ReyesPipeline(scene, flags=vp.FLAG_ONLINE)
    rp.configure(vp.HYBRID, vp.make_binding([(0, 1, vp.GROUP_MEGA, 0, split), (2, 3, vp.GROUP_RTC, split, nsm)], nsm))
    for _ in range(2):
        st = rp.run()
        check_against_oracle(orc, scene, rp, st)
        assert st["pending"] == 0 and st["abort_reason"] == 0
        assert sum(st["enqueued"][:4]) == sum(st["dequeued"][:4])
        if st["num_kernels"] > 2:  # the [Bound, Split] group retired before the end
            assert st["kernels"][2][:2] == (2, 3)
            assert sms_of(st["blocks_on_sm"][2]) <= set(range(split))


def test_toy_online_refill_happens(vpm, orc):
    """Fig. 9 toy, [S1] megakernel on 8 SMs | [S2, S3] RTC: the recursive S1 group drains
    first (nothing feeds it but its seeds), so its SMs must be refilled with S2/S3 blocks."""
    from paper_conf_micro_zhengozsyc17_b200.workloads import ToyPipeline
    vp = vpm
    nsm, _ = vp.device_info(0)
    seeds = inputs.toy_seeds(400_000)
    ref_out, ref_deq, _ = orc.toy_pipeline(seeds, inputs.TOY_THRESHOLD)
    tp = ToyPipeline(seeds, flags=vp.FLAG_ONLINE)
    tp.configure(vp.HYBRID, vp.make_binding([(0, 0, vp.GROUP_MEGA, 0, 8), (1, 2, vp.GROUP_RTC, 8, nsm)], nsm))
    refills = 0
    for _ in range(3):
        out, st = tp.run()
        assert np.array_equal(np.sort(out), np.sort(ref_out)) and st["dequeued"][:3] == ref_deq
        assert st["pending"] == 0
        if st["num_kernels"] == 3:
            refills += 1
            assert st["kernels"][2][:2] == (1, 2)
            assert sms_of(st["blocks_on_sm"][2]) <= set(range(8))
    assert refills >= 1


@pytest.mark.parametrize("model", ["pyramid", "facedet"])
def test_latched_workloads_online_parity(vpm, orc, model):
    """Latched pipelines under VP_FLAG_ONLINE: groups with cross-group feeders only retire
    after their feeders did; results stay bit-exact."""
    vp = vpm
    nsm, _ = vp.device_info(0)
    if model == "pyramid":
        from paper_conf_micro_zhengozsyc17_b200.workloads import PyramidPipeline
        from test_gpu_pyramid import check
        rgb = inputs.pyramid_images(2, 512)
        pp = PyramidPipeline(rgb, flags=vp.FLAG_ONLINE)
        pp.configure(vp.HYBRID, vp.make_binding([(0, 0, vp.GROUP_MEGA, 0, 100), (1, 3, vp.GROUP_MEGA, 100, nsm)], nsm))
        for _ in range(2):
            st = pp.run()
            check(orc, rgb, pp, st)
    else:
        from paper_conf_micro_zhengozsyc17_b200.workloads import FaceDetPipeline
        from test_gpu_facedet import check
        fs = inputs.face_scene(W=480, H=270)
        fp = FaceDetPipeline(fs, flags=vp.FLAG_ONLINE)
        fp.configure(vp.HYBRID, vp.make_binding([(0, 4, vp.GROUP_MEGA, 0, 40), (5, 5, vp.GROUP_MEGA, 40, nsm)], nsm))
        for _ in range(2):
            st = fp.run()
            check(orc, fs, fp, st)
    assert st["pending"] == 0 and st["abort_reason"] == 0


@pytest.mark.parametrize("model", ["hybrid", "megakernel", "kbk_graph"])
def test_reyes_l2_persist_parity(vpm, orc, model):
    """VP_FLAG_L2_PERSIST: the persisting window over the sequence words changes
    only cache residency, never results."""
    from paper_conf_micro_zhengozsyc17_b200.workloads import ReyesPipeline
    from test_gpu_reyes import check_against_oracle
    vp = vpm
    nsm, _ = vp.device_info(0)
    scene = inputs.reyes_config5(n_frames=8, n_side=16)
    rp = ReyesPipeline(scene, flags=vp.FLAG_L2_PERSIST)
    if model == "hybrid":
        rp.configure(vp.HYBRID, vp.make_binding([(0, 1, vp.GROUP_MEGA, 0, 60), (2, 3, vp.GROUP_RTC, 60, nsm)], nsm))
    else:
        rp.configure({"megakernel": vp.MEGAKERNEL, "kbk_graph": vp.KBK_GRAPH}[model])
    for _ in range(2):
        check_against_oracle(orc, scene, rp, rp.run())


def test_refill_goes_to_the_most_stalled_group(vpm, orc):
    """the freed SMs go to the group with stalled work.  Raster with
    [Vertex,Clip] (retires first), [Raster] and a deliberately small [Fragment] group: at
    the retirement Fragment holds far more live items than Raster, so the refill grid runs
    Fragment, not the first group downstream; the frame stays bit-exact."""
    from paper_conf_micro_zhengozsyc17_b200.workloads import RasterPipeline
    vp = vpm
    nsm, _ = vp.device_info(0)
    scene = inputs.raster_scene(200_000, W=1920, H=1080)
    rp = RasterPipeline(scene, flags=vp.FLAG_ONLINE)
    rp.configure(vp.HYBRID, vp.make_binding([(0, 1, vp.GROUP_RTC, 0, 40), (2, 2, vp.GROUP_MEGA, 40, 124),
                                             (3, 3, vp.GROUP_MEGA, 124, nsm)], nsm))
    ref = orc.raster_pipeline(scene)
    picked = []
    for _ in range(3):
        st = rp.run()
        assert np.array_equal(rp.keys(), ref["key"]) and np.array_equal(rp.colours(), ref["colour"])
        picked += [tuple(k[:2]) for k in st["kernels"][3:]]
    assert picked, "the [Vertex,Clip] group never retired before the end"
    assert all(k == (3, 3) for k in picked), picked

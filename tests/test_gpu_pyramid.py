"""GPU parity for the image pyramid (Fig. 12, L53; BASELINE config 3): bit-exact
pyramids, LUTs and per-stage counts against the CPU oracle, every execution model the
dependency latches allow."""
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


def configure(vp, pp, model):
    nsm, _ = vp.device_info(0)
    if model in ("kbk", "kbk_graph", "megakernel", "coarse", "fine"):
        pp.configure({"kbk": vp.KBK, "kbk_graph": vp.KBK_GRAPH, "megakernel": vp.MEGAKERNEL, "coarse": vp.COARSE, "fine": vp.FINE}[model])
    elif model == "hybrid":        # [Gray] mega | [CDF, Map, Resize] mega
        pp.configure(vp.HYBRID, vp.make_binding([(0, 0, vp.GROUP_MEGA, 0, 100), (1, 3, vp.GROUP_MEGA, 100, nsm)], nsm))
    elif model == "hybrid_kbk":    # [Gray] mega | [CDF] KBK | [Map, Resize] fine
        pp.configure(vp.HYBRID, vp.make_binding([(0, 0, vp.GROUP_MEGA, 0, 60), (1, 1, vp.GROUP_KBK, 60, 70),
                                                 (2, 3, vp.GROUP_FINE, 70, nsm)], nsm))
    else:
        raise ValueError(model)


def check(orc, rgb, pp, st):
    ref = orc.pyr_pipeline(rgb)
    got = pp.pyramid()
    assert np.array_equal(got, ref["pyr"]), f"{(got != ref['pyr']).sum()} pyramid bytes differ"
    assert np.array_equal(pp.lut.cpu().numpy(), ref["lut"])
    assert st["dequeued"][:4] == [ref["n_gray"], ref["n_cdf"], ref["n_map"], ref["n_resize"]]


@pytest.mark.parametrize("model", ["kbk", "kbk_graph", "megakernel", "coarse", "fine", "hybrid", "hybrid_kbk"])
def test_pyramid_reduced(vpm, orc, model):
    """512^2 x 2 images (SURVEY §8(d) reduced size)."""
    from paper_conf_micro_zhengozsyc17_b200.workloads import PyramidPipeline
    rgb = inputs.pyramid_images(2, 512)
    pp = PyramidPipeline(rgb)
    configure(vpm, pp, model)
    for _ in range(2):
        check(orc, rgb, pp, pp.run())


@pytest.mark.parametrize("S", [64, 128, 256])
def test_pyramid_small_levels(vpm, orc, S):
    from paper_conf_micro_zhengozsyc17_b200.workloads import PyramidPipeline
    rgb = inputs.pyramid_images(3, S)
    pp = PyramidPipeline(rgb)
    pp.configure(vpm.MEGAKERNEL)
    check(orc, rgb, pp, pp.run())


def test_pyramid_constant_image(vpm, orc):
    from paper_conf_micro_zhengozsyc17_b200.workloads import PyramidPipeline
    rgb = np.full((1, 256, 256, 3), 200, np.uint8)
    pp = PyramidPipeline(rgb)
    pp.configure(vpm.MEGAKERNEL)
    check(orc, rgb, pp, pp.run())


def test_pyramid_full_size(vpm, orc):
    """Config 3 image size (4096^2) on 2 images, in the megakernel launch configuration."""
    from paper_conf_micro_zhengozsyc17_b200.workloads import PyramidPipeline
    rgb = inputs.pyramid_images(2, 4096)
    pp = PyramidPipeline(rgb)
    pp.configure(vpm.MEGAKERNEL)
    check(orc, rgb, pp, pp.run())


@pytest.mark.parametrize("model", ["kbk", "kbk_graph"])
def test_pyramid_kbk_with_streams(vpm, orc, model):
    """The "KBK with Stream" baseline (L53-L55, Fig. 13): images split over concurrent
    per-stream KBK pipelines (one host thread each) give the same pyramids."""
    import torch
    from paper_conf_micro_zhengozsyc17_b200.workloads import PyramidKbkStreams
    vp = vpm
    rgb = inputs.pyramid_images(5, 256)
    ks = PyramidKbkStreams(torch.from_numpy(rgb).cuda(), 3, model=vp.KBK if model == "kbk" else vp.KBK_GRAPH)
    assert ks.n_streams == 3
    for _ in range(2):
        ks.run()
        torch.cuda.synchronize()
        assert np.array_equal(ks.pyramid(), orc.pyr_pipeline(rgb)["pyr"])

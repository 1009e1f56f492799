"""GPU parity for LBP face detection (Fig. 14, L55; BASELINE config 2): the detection set
(item-id-sorted multiset), per-cascade-stage survivor counts, the windows evaluated
(5 306 934 per 1080p frame), the equalised pyramid, LBP codes and per-stage task counts
are bit-exact against the CPU oracle under every legal execution model."""
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


def configure(vp, fp, model):
    nsm, _ = vp.device_info(0)
    if model in ("kbk", "kbk_graph", "megakernel", "coarse", "fine"):
        fp.configure({"kbk": vp.KBK, "kbk_graph": vp.KBK_GRAPH, "megakernel": vp.MEGAKERNEL, "coarse": vp.COARSE, "fine": vp.FINE}[model])
    elif model == "hybrid":      # [Gray..LBP] megakernel | [Scan] fine on most SMs
        fp.configure(vp.HYBRID, vp.make_binding([(0, 4, vp.GROUP_MEGA, 0, 40), (5, 5, vp.GROUP_MEGA, 40, nsm)], nsm))
    elif model == "hybrid_kbk":  # [Gray] mega | [CDF] KBK | [Map..Scan] mega
        fp.configure(vp.HYBRID, vp.make_binding([(0, 0, vp.GROUP_MEGA, 0, 30), (1, 1, vp.GROUP_KBK, 30, 40),
                                                 (2, 5, vp.GROUP_MEGA, 40, nsm)], nsm))
    elif model == "hybrid_rtc":  # [Gray..Resize] mega | [LBP, Scan] RTC: Scan runs LBP's 64-row local batches
        fp.configure(vp.HYBRID, vp.make_binding([(0, 3, vp.GROUP_MEGA, 0, 40), (4, 5, vp.GROUP_RTC, 40, nsm)], nsm))
    else:
        raise ValueError(model)


def check(orc, sc, fp, st):
    ref = orc.fd_pipeline(sc, det_cap=1 << 20)
    got = fp.results()
    assert got["n_det"] == ref["n_det"]
    a = sorted(map(tuple, got["det"].tolist()))
    b = sorted(map(tuple, ref["det"].astype(np.int64).tolist()))
    assert a == b
    assert got["survivors"] == ref["survivors"] and got["windows"] == ref["windows"]
    assert np.array_equal(fp.levels.cpu().numpy(), ref["levels"])
    assert np.array_equal(fp.lbp.cpu().numpy(), ref["lbp"])
    assert st["dequeued"][:6] == ref["deq"]


@pytest.mark.parametrize("model", ["kbk", "kbk_graph", "megakernel", "coarse", "fine", "hybrid", "hybrid_kbk",
                                   "hybrid_rtc"])
def test_facedet_reduced(vpm, orc, model):
    """480x270 frame (SURVEY §8(d) reduced size), 2 frames."""
    from paper_conf_micro_zhengozsyc17_b200.workloads import FaceDetPipeline
    sc = inputs.face_scene(W=480, H=270, n_frames=2, n_planted=6)
    fp = FaceDetPipeline(sc)
    configure(vpm, fp, model)
    for _ in range(2):
        check(orc, sc, fp, fp.run())


@pytest.mark.parametrize("model", ["megakernel", "hybrid_rtc"])
def test_facedet_full_frame(vpm, orc, model):
    """Config 2: 1920x1080, 8 levels, 5 306 934 windows, in the megakernel configuration
    and with an RTC [LBP, Scan] group (Scan batches of up to 128 block-local rows)."""
    from paper_conf_micro_zhengozsyc17_b200.workloads import FaceDetPipeline
    sc = inputs.face_scene()
    fp = FaceDetPipeline(sc)
    configure(vpm, fp, model)
    st = fp.run()
    check(orc, sc, fp, st)
    assert fp.results()["windows"] == 5_306_934

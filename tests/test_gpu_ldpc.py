"""GPU parity for the LDPC decoder (Fig. 17, L59): posteriors,
per-iteration bit-error counts and stage counts (chunked items, reading R-L6) bit-exact
against the CPU oracle under every execution model, including the paper's hybrid
([Initialize, C2V] fine | [V2C] | [ProbVar]) and the full 100 frames x 100 iterations."""
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


def configure(vp, lp, model):
    nsm, _ = vp.device_info(0)
    if model in ("kbk", "kbk_graph", "megakernel", "coarse", "fine"):
        lp.configure({"kbk": vp.KBK, "kbk_graph": vp.KBK_GRAPH, "megakernel": vp.MEGAKERNEL, "coarse": vp.COARSE,
                      "fine": vp.FINE}[model])
    elif model == "hybrid_paper":   # L59: Initialize and C2V in a fine group, V2C and ProbVar megakernels
        lp.configure(vp.HYBRID, vp.make_binding([(0, 1, vp.GROUP_FINE, 0, 60), (2, 2, vp.GROUP_MEGA, 60, 104),
                                                 (3, 3, vp.GROUP_MEGA, 104, nsm)], nsm))
    elif model == "hybrid_rtc":     # [Initialize] RTC | [C2V, V2C, ProbVar] megakernel
        lp.configure(vp.HYBRID, vp.make_binding([(0, 0, vp.GROUP_RTC, 0, 20), (1, 3, vp.GROUP_MEGA, 20, nsm)], nsm))
    else:
        raise ValueError(model)


def check(orc, sc, lp, st):
    ref = orc.ldpc_pipeline(sc)
    got = lp.results()
    assert np.array_equal(got["post"], ref["post"])
    assert np.array_equal(got["errors"], ref["errors"])
    assert st["dequeued"][:4] == ref["deq"]


@pytest.mark.parametrize("model", ["kbk", "kbk_graph", "megakernel", "coarse", "fine", "hybrid_paper", "hybrid_rtc"])
def test_ldpc_reduced(vpm, orc, model):
    from paper_conf_micro_zhengozsyc17_b200.workloads import LdpcPipeline
    sc = inputs.ldpc_scene(n_frames=16, n_iter=20)
    lp = LdpcPipeline(sc)
    configure(vpm, lp, model)
    for _ in range(2):
        check(orc, sc, lp, lp.run())


@pytest.mark.parametrize("batch", [1, 2, 4])
def test_ldpc_batches(vpm, orc, batch):
    from paper_conf_micro_zhengozsyc17_b200.workloads import LdpcPipeline
    sc = inputs.ldpc_scene(n_frames=9, n_iter=7, ebn0_db=1.5)
    lp = LdpcPipeline(sc)
    lp.configure(vpm.MEGAKERNEL, None, batch)
    check(orc, sc, lp, lp.run())


def test_ldpc_generic_degrees(vpm, orc):
    """A (4, 8)-regular code exercises the run-time-degree paths."""
    from paper_conf_micro_zhengozsyc17_b200.workloads import LdpcPipeline
    sc = inputs.ldpc_scene(n_frames=4, N=512, dv=4, dc=8, n_iter=6)
    lp = LdpcPipeline(sc)
    lp.configure(vpm.MEGAKERNEL)
    check(orc, sc, lp, lp.run())


def test_ldpc_full_size(vpm, orc):
    """The paper's size: 100 frames x 100 iterations (L53)."""
    from paper_conf_micro_zhengozsyc17_b200.workloads import LdpcPipeline
    sc = inputs.ldpc_scene()
    lp = LdpcPipeline(sc)
    configure(vpm, lp, "hybrid_paper")
    check(orc, sc, lp, lp.run())

"""GPU parity for the CFD solver (Fig. 15, L55; BASELINE config 3): bit-exact final state
(<= 1e-4 stated, bit-exact expected) and per-stage counts against the CPU oracle under
the execution models its loop allows; free-stream fixed point on the GPU."""
import numpy as np
import pytest

from paper_conf_micro_zhengozsyc17_b200 import inputs

pytestmark = pytest.mark.gpu
TOL = 1e-4


@pytest.fixture(scope="module")
def vpm():
    import torch
    if not torch.cuda.is_available():
        pytest.skip("needs a GPU")
    from paper_conf_micro_zhengozsyc17_b200 import vp
    return vp


def configure(vp, cp, model):
    nsm, _ = vp.device_info(0)
    if model in ("kbk", "kbk_graph", "megakernel", "coarse", "fine"):
        cp.configure({"kbk": vp.KBK, "kbk_graph": vp.KBK_GRAPH, "megakernel": vp.MEGAKERNEL, "coarse": vp.COARSE, "fine": vp.FINE}[model])
    elif model == "hybrid":           # [Copy, StepFactor] RTC | [Flux, TimeStep] megakernel
        cp.configure(vp.HYBRID, vp.make_binding([(0, 1, vp.GROUP_RTC, 0, 24), (2, 3, vp.GROUP_MEGA, 24, nsm)], nsm))
    elif model == "hybrid_fine":      # [Copy, StepFactor] mega | [Flux, TimeStep] fine
        cp.configure(vp.HYBRID, vp.make_binding([(0, 1, vp.GROUP_MEGA, 0, 24), (2, 3, vp.GROUP_FINE, 24, nsm)], nsm))
    else:
        raise ValueError(model)


def check(orc, sc, cp, st):
    ref = orc.cfd_pipeline(sc)
    got = cp.state()
    assert np.max(np.abs(got - ref["vars"])) <= TOL
    assert np.array_equal(got, ref["vars"]), f"{(got != ref['vars']).sum()} values differ"
    assert st["dequeued"][:4] == [ref["n_copy"], ref["n_step"], ref["n_flux"], ref["n_time"]]


@pytest.mark.parametrize("model", ["kbk", "kbk_graph", "megakernel", "coarse", "fine", "hybrid", "hybrid_fine"])
def test_cfd_64_two_iterations(vpm, orc, model):
    from paper_conf_micro_zhengozsyc17_b200.workloads import CfdPipeline
    sc = inputs.cfd_scene(G=64, n_outer=2)
    cp = CfdPipeline(sc)
    configure(vpm, cp, model)
    for _ in range(2):
        check(orc, sc, cp, cp.run())


def test_cfd_256_ten_iterations(vpm, orc):
    from paper_conf_micro_zhengozsyc17_b200.workloads import CfdPipeline
    sc = inputs.cfd_scene(G=256, n_outer=10)
    cp = CfdPipeline(sc)
    configure(vpm, cp, "megakernel")
    check(orc, sc, cp, cp.run())


def test_cfd_free_stream_fixed_point(vpm):
    from paper_conf_micro_zhengozsyc17_b200.workloads import CfdPipeline
    sc = inputs.cfd_scene(G=128, n_outer=3, uniform=True)
    cp = CfdPipeline(sc)
    configure(vpm, cp, "megakernel")
    cp.run()
    assert np.array_equal(cp.state(), sc.vars0)


def test_cfd_full_grid_one_iteration(vpm, orc):
    """Config 3 grid (4096^2, 1024-cell tiles), one outer iteration: all cells compared."""
    from paper_conf_micro_zhengozsyc17_b200.workloads import CfdPipeline
    sc = inputs.cfd_scene(G=4096, n_outer=1)
    cp = CfdPipeline(sc)
    configure(vpm, cp, "megakernel")
    check(orc, sc, cp, cp.run())

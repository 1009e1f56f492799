"""GPU parity for Reyes (Fig. 1, L3; L55): every execution model through the C ABI,
bit-exact depth keys / shade factors / colours (tolerance 1e-4 stated by north_star,
bit-exact expected under -fmad=false), per-stage counts and the (stage, node id)
trace multiset against the CPU oracle."""
import numpy as np
import pytest

from paper_conf_micro_zhengozsyc17_b200 import inputs

pytestmark = pytest.mark.gpu
TOL = 1e-4   # north_star: shaded pixels within max abs error 1e-4


@pytest.fixture(scope="module")
def vpm():
    import torch
    if not torch.cuda.is_available():
        pytest.skip("needs a GPU")
    from paper_conf_micro_zhengozsyc17_b200 import vp
    return vp


def configure(vp, rp, model):
    nsm, _ = vp.device_info(0)
    h = nsm // 2
    if model == "kbk":
        rp.configure(vp.KBK)
    elif model == "kbk_graph":            # KBK with the wave loop in a CUDA-graph while node
        rp.configure(vp.KBK_GRAPH)
    elif model == "megakernel":
        rp.configure(vp.MEGAKERNEL)
    elif model == "coarse":
        rp.configure(vp.COARSE)
    elif model == "fine":
        rp.configure(vp.FINE)
    elif model == "hybrid_mega_rtc":      # [Bound,Split] megakernel | [Dice,Shade] RTC
        rp.configure(vp.HYBRID, vp.make_binding([(0, 1, vp.GROUP_MEGA, 0, h), (2, 3, vp.GROUP_RTC, h, nsm)], nsm))
    elif model == "hybrid_fine_rtc":      # [Bound,Split] fine | [Dice,Shade] RTC
        rp.configure(vp.HYBRID, vp.make_binding([(0, 1, vp.GROUP_FINE, 0, 40), (2, 3, vp.GROUP_RTC, 40, nsm)], nsm))
    elif model == "hybrid_kbk":           # [Bound,Split] megakernel | [Dice] KBK | [Shade] fine
        rp.configure(vp.HYBRID, vp.make_binding([(0, 1, vp.GROUP_MEGA, 0, 50), (2, 2, vp.GROUP_KBK, 50, 90),
                                                 (3, 3, vp.GROUP_FINE, 90, nsm)], nsm))
    elif model == "hybrid_4":             # each stage its own group: coarse pipeline of groups
        rp.configure(vp.HYBRID, vp.make_binding([(0, 0, vp.GROUP_MEGA, 0, 30), (1, 1, vp.GROUP_MEGA, 30, 50),
                                                 (2, 2, vp.GROUP_MEGA, 50, 100), (3, 3, vp.GROUP_MEGA, 100, nsm)], nsm))
    elif model == "hybrid_mega_rtc3":     # [Bound] megakernel | [Split,Dice,Shade] RTC (fused Dice batches)
        rp.configure(vp.HYBRID, vp.make_binding([(0, 0, vp.GROUP_MEGA, 0, 24), (1, 3, vp.GROUP_RTC, 24, nsm)], nsm,
                                                batch=[32, 16, 32, 4]))
    else:
        raise ValueError(model)


def check_against_oracle(orc, scene, rp, st, trace=None):
    ref = orc.reyes_pipeline(scene, trace_cap=1 << 22)
    key, s = rp.keys()
    assert np.array_equal(key, ref["key"]), f"{(key != ref['key']).sum()} pixel keys differ"
    assert np.array_equal(s, ref["s"])
    col = rp.colours()
    assert np.max(np.abs(col - ref["colour"])) <= TOL
    assert np.array_equal(col, ref["colour"])      # bit-exact is the expectation (-fmad=false)
    assert st["dequeued"][:4] == [ref["n_bound"], ref["n_split"], ref["n_dice"], ref["n_shade"]]
    if trace is not None:
        rt = ref["trace"]
        for stage in range(4):
            a = np.sort(trace["id"][trace["stage"] == stage])
            b = np.sort(rt["id"][rt["stage"] == stage])
            assert np.array_equal(a, b), f"stage {stage} trace multiset differs"
    return ref


MODELS = ["kbk", "kbk_graph", "megakernel", "coarse", "fine", "hybrid_mega_rtc", "hybrid_fine_rtc", "hybrid_kbk", "hybrid_4",
          "hybrid_mega_rtc3"]


@pytest.mark.parametrize("model", MODELS)
def test_reyes_config1_all_models(vpm, orc, model):
    from paper_conf_micro_zhengozsyc17_b200.workloads import ReyesPipeline
    scene = inputs.reyes_config1()
    rp = ReyesPipeline(scene)
    configure(vpm, rp, model)
    for _ in range(2):
        st = rp.run()
        check_against_oracle(orc, scene, rp, st)


def test_reyes_rtc_rejected(vpm):
    from paper_conf_micro_zhengozsyc17_b200.workloads import ReyesPipeline
    vp = vpm
    rp = ReyesPipeline(inputs.reyes_config1())
    with pytest.raises(vp.VPError) as e:
        rp.configure(vp.RTC)          # Split -> Bound recursion (L55: RTC impractical for Reyes)
    assert e.value.status == vp.VP_ERR_UNSUPPORTED
    nsm, _ = vp.device_info(0)
    with pytest.raises(vp.VPError) as e:
        rp.configure(vp.HYBRID, vp.make_binding([(0, 1, vp.GROUP_RTC, 0, 70), (2, 3, vp.GROUP_RTC, 70, nsm)], nsm))
    assert e.value.status == vp.VP_ERR_UNSUPPORTED


@pytest.mark.parametrize("model", ["megakernel", "hybrid_mega_rtc", "kbk", "kbk_graph"])
def test_reyes_trace_multiset(vpm, orc, model):
    """Each (stage, node) is dequeued exactly once and the multiset equals the oracle's."""
    from paper_conf_micro_zhengozsyc17_b200.workloads import ReyesPipeline
    vp = vpm
    scene = inputs.reyes_config1()
    rp = ReyesPipeline(scene, flags=vp.FLAG_TRACE, trace_capacity=1 << 16)
    configure(vp, rp, model)
    st = rp.run()
    tr = trace_array(rp, st)
    check_against_oracle(orc, scene, rp, st, trace=tr)


def trace_array(rp, st):
    """The library trace buffer (device) through the binding's memcpy."""
    return rp.p.trace(st)


@pytest.mark.parametrize("batch", [1, 3, 8])
def test_reyes_batch_sizes(vpm, orc, batch):
    from paper_conf_micro_zhengozsyc17_b200.workloads import ReyesPipeline
    vp = vpm
    scene = inputs.reyes_config1()
    rp = ReyesPipeline(scene)
    rp.configure(vp.MEGAKERNEL, None, batch)
    check_against_oracle(orc, scene, rp, rp.run())


@pytest.mark.parametrize("model", ["megakernel", "hybrid_mega_rtc", "kbk", "kbk_graph"])
def test_reyes_config5_reduced(vpm, orc, model):
    """Config 5 at CI size: 8 frames x 256 patches (SURVEY §8(d) reduced sizes)."""
    from paper_conf_micro_zhengozsyc17_b200.workloads import ReyesPipeline
    scene = inputs.reyes_config5(n_frames=8, n_side=16)
    rp = ReyesPipeline(scene)
    configure(vpm, rp, model)
    check_against_oracle(orc, scene, rp, rp.run())


def test_reyes_planar_closed_form(vpm, orc):
    from paper_conf_micro_zhengozsyc17_b200.workloads import ReyesPipeline
    vp = vpm
    scene = inputs.reyes_planar(48.0, W=64, H=64, x0=8.5, y0=8.5)
    rp = ReyesPipeline(scene)
    rp.configure(vp.MEGAKERNEL)
    st = rp.run()
    key, _ = rp.keys()
    cov = key[0] != np.uint64(0xFFFFFFFFFFFFFFFF)
    exp = np.zeros((64, 64), bool)
    exp[9:57, 9:57] = True
    assert np.array_equal(cov, exp)
    assert st["dequeued"][2] == 64


def test_reyes_full_config5_sampled_frames(vpm, orc):
    """Full config 5 shape (4096 patches/frame) on a 16-frame shard, in the launch
    configuration bench.py times (hybrid); frames sampled for the oracle."""
    from paper_conf_micro_zhengozsyc17_b200.workloads import ReyesPipeline
    vp = vpm
    scene = inputs.reyes_config5(n_frames=16)
    rp = ReyesPipeline(scene)
    configure(vp, rp, "hybrid_mega_rtc")
    st = rp.run()
    key, s = rp.keys()
    col = rp.colours()
    tot = [0, 0, 0, 0]
    for f in (0, 7, 15):
        sub = inputs.reyes_config5(n_frames=1, frame0=f)
        ref = orc.reyes_pipeline(sub)
        assert np.array_equal(key[f], ref["key"][0]) and np.array_equal(col[f], ref["colour"][0])
    # whole-shard conservation (any size): Bound = seeds + 2 Split; Shade = Dice
    d = st["dequeued"]
    assert d[0] == scene.seeds.size + 2 * d[1] and d[3] == d[2]


def test_reyes_config1_throughput_mode_replicas(vpm, orc):
    """SURVEY §8(d) throughput mode: R replicated config-1 frames in one run; every frame
    equals the single-frame oracle result."""
    from paper_conf_micro_zhengozsyc17_b200.workloads import ReyesPipeline
    scene = inputs.reyes_config1(n_frames=4)
    rp = ReyesPipeline(scene)
    configure(vpm, rp, "hybrid_mega_rtc")
    check_against_oracle(orc, scene, rp, rp.run())


@pytest.mark.parametrize("model", ["megakernel", "hybrid_mega_rtc", "kbk_graph"])
def test_reyes_config1_x256_wide_recursion(vpm, orc, model):
    """256 replicas of config 1 recurse all at once (a frontier of thousands of deep split
    trees): the recursive rings of the block-local [Bound, Split] kernel must hold it (no
    VP_ERR_QUEUE_OVERFLOW), and every replica equals the single-frame oracle."""
    from paper_conf_micro_zhengozsyc17_b200.workloads import ReyesPipeline
    one = inputs.reyes_config1()
    ref = orc.reyes_pipeline(one)
    scene = inputs.reyes_config1(n_frames=256)
    rp = ReyesPipeline(scene)
    configure(vpm, rp, model)
    st = rp.run()
    assert st["dequeued"][:4] == [256 * ref["n_bound"], 256 * ref["n_split"], 256 * ref["n_dice"], 256 * ref["n_shade"]]
    key, _ = rp.keys()
    col = rp.colours()
    for f in (0, 1, 77, 255):
        assert np.array_equal(key[f], ref["key"][0]) and np.array_equal(col[f], ref["colour"][0])


@pytest.mark.parametrize("model", ["hybrid_mega_rtc", "megakernel"])
def test_reyes_stream_host_buffers(vpm, orc, model):
    """The e2e path (workloads.ReyesStream): chunks of frames re-targeted with vp_set_params
    (frame_base, matrices) and rendered from pinned host buffers by two pipelines in turn,
    with copies overlapping runs, twice over the batch; every frame equals the resident
    single-pipeline render and the oracle."""
    import torch
    from paper_conf_micro_zhengozsyc17_b200.workloads import ReyesPipeline, ReyesStream
    scene = inputs.reyes_config5(n_frames=16, n_side=16)
    rp = ReyesPipeline(scene)
    configure(vpm, rp, model)
    rp.run()
    want = rp.colours()
    rs = ReyesStream(scene, chunk=4)
    for p in rs.pipes:
        configure(vpm, p, model)
    host_seeds = ReyesStream.host_seeds(scene)
    host_M = torch.from_numpy(np.ascontiguousarray(scene.M, np.float32)).pin_memory()
    host_out = torch.full((16, scene.H, scene.W, 4), -1.0).pin_memory()
    rs.render(host_seeds, host_M, host_out, steps=2)
    torch.cuda.synchronize()
    got = host_out.numpy()
    assert np.array_equal(got, want)
    for f in (0, 9):
        ref = orc.reyes_pipeline(inputs.reyes_config5(n_frames=1, n_side=16, frame0=f))
        assert np.array_equal(got[f], ref["colour"][0])


@pytest.mark.parametrize("model", ["hybrid_mega_rtc", "megakernel"])
def test_shade_work_units_match_oracle(vpm, orc, model):
    """The micropolygons the fused [Dice, Shade] chain reports shading
    (vp_run_stats.work_units[Shade], the count bench.py's roofline uses) equal the oracle's
    count of micropolygons whose screen box holds a pixel centre."""
    from paper_conf_micro_zhengozsyc17_b200.workloads import ReyesPipeline
    for scene in (inputs.reyes_config1(), inputs.reyes_config5(n_frames=8, n_side=16)):
        rp = ReyesPipeline(scene)
        configure(vpm, rp, model)
        st = rp.run()
        ref = orc.reyes_pipeline(scene)
        assert st["work_units"][3] == ref["n_mp_covering"] > 0

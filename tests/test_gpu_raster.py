"""GPU parity for rasterization (Fig. 16, L59; BASELINE config 4) through the C ABI:
bit-exact depth keys, colours (<= 1e-4, bit-exact expected), per-stage counts and the
trace multiset against the CPU oracle, under every legal execution model."""
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


def configure(vp, rp, model):
    nsm, _ = vp.device_info(0)
    if model in ("kbk", "kbk_graph", "megakernel", "coarse", "fine"):
        rp.configure({"kbk": vp.KBK, "kbk_graph": vp.KBK_GRAPH, "megakernel": vp.MEGAKERNEL, "coarse": vp.COARSE, "fine": vp.FINE}[model])
    elif model == "hybrid_rtc_mega":      # [Vertex,Clip] RTC (the paper's Clip) | [Raster,Fragment] megakernel
        rp.configure(vp.HYBRID, vp.make_binding([(0, 1, vp.GROUP_RTC, 0, 40), (2, 3, vp.GROUP_MEGA, 40, nsm)], nsm))
    elif model == "hybrid_rtc_rtc":       # [Vertex,Clip] RTC | [Raster,Fragment] RTC
        rp.configure(vp.HYBRID, vp.make_binding([(0, 1, vp.GROUP_RTC, 0, 40), (2, 3, vp.GROUP_RTC, 40, nsm)], nsm))
    elif model == "hybrid_fine":          # [Vertex..Raster] megakernel | [Fragment] fine
        rp.configure(vp.HYBRID, vp.make_binding([(0, 2, vp.GROUP_MEGA, 0, 30), (3, 3, vp.GROUP_FINE, 30, nsm)], nsm))
    else:
        raise ValueError(model)


def check(orc, scene, rp, st):
    ref = orc.raster_pipeline(scene)
    key = rp.keys()
    assert np.array_equal(key, ref["key"]), f"{(key != ref['key']).sum()} keys differ"
    col = rp.colours()
    assert np.max(np.abs(col - ref["colour"])) <= TOL
    assert np.array_equal(col, ref["colour"])
    assert st["dequeued"][:4] == [ref["n_vertex"], ref["n_clip"], ref["n_raster"], ref["n_fragment"]]
    return ref


MODELS = ["kbk", "kbk_graph", "megakernel", "coarse", "fine", "hybrid_rtc_mega", "hybrid_rtc_rtc", "hybrid_fine"]


@pytest.mark.parametrize("model", MODELS)
def test_raster_reduced(vpm, orc, model):
    """10^4 triangles at 320x180 (SURVEY §8(d) reduced size)."""
    from paper_conf_micro_zhengozsyc17_b200.workloads import RasterPipeline
    scene = inputs.raster_scene(10_000, W=320, H=180)
    rp = RasterPipeline(scene)
    configure(vpm, rp, model)
    for _ in range(2):
        check(orc, scene, rp, rp.run())


def test_raster_rtc_whole_pipeline_rejected(vpm):
    from paper_conf_micro_zhengozsyc17_b200.workloads import RasterPipeline
    vp = vpm
    rp = RasterPipeline(inputs.raster_scene(100, W=64, H=64))
    with pytest.raises(vp.VPError) as e:
        rp.configure(vp.RTC)   # Raster's fan-out cannot be expanded block-locally
    assert e.value.status == vp.VP_ERR_UNSUPPORTED


def test_raster_tiny_brute_force_scene(vpm, orc):
    from paper_conf_micro_zhengozsyc17_b200.workloads import RasterPipeline
    vp = vpm
    scene = inputs.raster_scene(200, W=64, H=64, seed=inputs.seed_for(4, 1), area_range=(0.5, 200.0))
    rp = RasterPipeline(scene)
    rp.configure(vp.MEGAKERNEL)
    check(orc, scene, rp, rp.run())


def test_raster_watertight(vpm, orc):
    from paper_conf_micro_zhengozsyc17_b200.workloads import RasterPipeline
    vp = vpm
    scene = inputs.raster_quad_mesh(320, 176, cell=16)
    rp = RasterPipeline(scene)
    rp.configure(vp.MEGAKERNEL)
    check(orc, scene, rp, rp.run())
    assert np.all(rp.keys() != np.uint64(0xFFFFFFFFFFFFFFFF))


def test_raster_full_config4_sampled(vpm, orc):
    """Full config 4 (1M triangles, 1920x1080) in the hybrid launch configuration; the
    oracle runs the whole frame (~5 s) and everything is compared."""
    from paper_conf_micro_zhengozsyc17_b200.workloads import RasterPipeline
    scene = inputs.raster_scene()
    rp = RasterPipeline(scene)
    configure(vpm, rp, "hybrid_rtc_mega")
    check(orc, scene, rp, rp.run())


def _merge_local(parts):
    """raster_merge's exchange step on one device: MIN of the order-preserving keys, then
    the colour of the rank that holds the winning key."""
    import torch
    from paper_conf_micro_zhengozsyc17_b200 import shard
    ks = [shard.ukey_to_ordered(k) for k, _ in parts]
    kmin = ks[0]
    for k in ks[1:]:
        kmin = torch.minimum(kmin, k)
    col = sum(torch.where((k == kmin).unsqueeze(-1), c, torch.zeros_like(c)) for k, (_, c) in zip(ks, parts))
    return shard.ukey_to_ordered(kmin), col


@pytest.mark.parametrize("shards", [2, 4])
def test_raster_triangle_shards_merge_bit_exact(vpm, orc, shards):
    """the frame rendered as `shards` triangle shards (each a pipeline run
    over its id range, as one rank would) and merged by the MIN-key exchange equals the
    oracle (reduced scene) and the unsharded GPU frame (full 1M-triangle config 4)."""
    from paper_conf_micro_zhengozsyc17_b200 import shard
    from paper_conf_micro_zhengozsyc17_b200.workloads import RasterPipeline
    vp = vpm
    for sc, ref_fn in ((inputs.raster_scene(n=10_000, W=320, H=180), "oracle"), (inputs.raster_scene(), "gpu")):
        parts = []
        for r in range(shards):
            lo, hi = shard.shard_range(r, shards, sc.n_tris)
            rp = RasterPipeline(sc, tri_range=(lo, hi))
            rp.configure(vp.MEGAKERNEL)
            rp.run()
            parts.append((rp.fb.clone(), rp.colour.clone()))
            del rp
        k, c = _merge_local(parts)
        if ref_fn == "oracle":
            ref = orc.raster_definition(sc)
            rk, rc = ref["key"], ref["colour"]
        else:
            full = RasterPipeline(sc)
            full.configure(vp.MEGAKERNEL)
            full.run()
            rk, rc = full.keys(), full.colour.cpu().numpy()
        assert np.array_equal(k.cpu().numpy().view(np.uint64), rk.reshape(k.shape))
        assert np.array_equal(c.cpu().numpy(), rc.reshape(c.shape))


@pytest.mark.parametrize("model", MODELS)
def test_raster_near_clip(vpm, orc, model):
    """Near-plane clipping (DESIGN R-S9): Clip fans out 0..2 sub-triangles;
    keys (sub-ids 2 tri + j), colours and per-stage counts bit-exact with the oracle."""
    from paper_conf_micro_zhengozsyc17_b200.workloads import RasterPipeline
    scene = inputs.raster_near_scene(4096, W=256, H=192)
    rp = RasterPipeline(scene)
    configure(vpm, rp, model)
    for _ in range(2):
        ref = check(orc, scene, rp, rp.run())
    assert ref["n_raster"] > ref["n_clip"] // 2  # sub-triangles were emitted


@pytest.mark.parametrize("model", ["kbk", "megakernel", "hybrid_rtc_mega"])
def test_raster_near_clip_perspective(vpm, orc, model):
    """Perspective scene (w = z + 0.5, some vertices at w <= 0): the clipped sub-triangles
    have interpolated w; bit-exact with the oracle."""
    from paper_conf_micro_zhengozsyc17_b200.workloads import RasterPipeline
    scene = inputs.raster_near_scene(4096, W=256, H=192, z_range=(-0.9, 0.95), perspective=True)
    rp = RasterPipeline(scene)
    configure(vpm, rp, model)
    check(orc, scene, rp, rp.run())


def test_raster_near_clip_off_matches_default(vpm, orc):
    """near_clip = 1 on a scene with no vertex behind z = 0 renders the default image with
    every key's id doubled (the clip is the identity there)."""
    from paper_conf_micro_zhengozsyc17_b200.workloads import RasterPipeline
    scene = inputs.raster_scene(3000, W=256, H=192)
    a = RasterPipeline(scene)
    a.configure(vpm.MEGAKERNEL)
    a.run()
    scene.near_clip = 1
    b = RasterPipeline(scene)
    b.configure(vpm.MEGAKERNEL)
    b.run()
    ka, kb = a.keys(), b.keys()
    hit = ka != np.uint64(0xFFFFFFFFFFFFFFFF)
    assert np.array_equal(hit, kb != np.uint64(0xFFFFFFFFFFFFFFFF))
    assert np.array_equal(ka[hit] >> np.uint64(32), kb[hit] >> np.uint64(32))
    assert np.array_equal((ka[hit] & np.uint64(0xFFFFFFFF)) * np.uint64(2), kb[hit] & np.uint64(0xFFFFFFFF))
    assert np.array_equal(a.colours(), b.colours())


@pytest.mark.parametrize("model", ["hybrid_rtc_rtc", "megakernel"])
def test_raster_near_clip_full_size(vpm, orc, model):
    """The bench's near-clip workload at full size (1M triangles, 1920x1080, about half
    straddling z = 0) against the whole-frame oracle (~5 s), bit-exact."""
    from paper_conf_micro_zhengozsyc17_b200.workloads import RasterPipeline
    scene = inputs.raster_near_scene(n=1 << 20, W=1920, H=1080, area_range=(0.5, 512.0))
    rp = RasterPipeline(scene)
    configure(vpm, rp, model)
    check(orc, scene, rp, rp.run())


def test_raster_near_clip_shards_merge_bit_exact(vpm, orc):
    """Triangle shards with near clipping: sub-ids 2 tri + j stay global,
    so the MIN-key merge of 3 shards equals the oracle's frame."""
    from paper_conf_micro_zhengozsyc17_b200 import shard
    from paper_conf_micro_zhengozsyc17_b200.workloads import RasterPipeline
    sc = inputs.raster_near_scene(4096, W=256, H=192, z_range=(-0.9, 0.95), perspective=True)
    parts = []
    for r in range(3):
        lo, hi = shard.shard_range(r, 3, sc.n_tris)
        rp = RasterPipeline(sc, tri_range=(lo, hi))
        rp.configure(vpm.MEGAKERNEL)
        rp.run()
        parts.append((rp.fb.clone(), rp.colour.clone()))
    k, c = _merge_local(parts)
    ref = orc.raster_definition(sc)
    assert np.array_equal(k.cpu().numpy().view(np.uint64), ref["key"].reshape(k.shape))
    assert np.array_equal(c.cpu().numpy(), ref["colour"].reshape(c.shape))


@pytest.mark.parametrize("zs", [(-0.2, 0.3, 0.4), (0.2, -0.3, 0.4), (0.2, 0.3, -0.4), (-0.2, -0.3, 0.4),
                                (0.2, -0.3, -0.4), (-0.2, 0.3, -0.4), (0.2, 0.3, 0.4)])
def test_raster_near_clip_every_side_pattern(vpm, orc, zs):
    """One triangle per in/out pattern of its vertices (the polygon's 4th vertex is an
    original vertex only for in-out-in), under both vertex orders, bit-exact."""
    from paper_conf_micro_zhengozsyc17_b200.workloads import RasterPipeline
    for order in ((0, 1, 2), (0, 2, 1)):
        xy = [(8, 8), (56, 10), (30, 56)]
        pos = np.zeros((1, 3, 4), np.float32)
        col = np.zeros((1, 3, 4), np.float32)
        for k, o in enumerate(order):
            pos[0, k] = (*xy[o], zs[o], 1.0)
            col[0, k, :3] = np.eye(3)[o]
        scene = inputs.RasterScene(W=64, H=64, M=inputs.pixel_to_ndc(64, 64), pos=pos, col=col, near_clip=1)
        rp = RasterPipeline(scene)
        rp.configure(vpm.MEGAKERNEL)
        check(orc, scene, rp, rp.run())


def _with_big_triangles(sc, straddle):
    """Prepend screen-filling triangles (beyond the 128-tile fan-out): a
    full-screen quad at z = 0.9 and a 3-screen-wide triangle; with `straddle` one vertex of
    each lies behind the near plane (z < 0), so the clipped pieces are big as well."""
    import dataclasses
    W, H = sc.W, sc.H
    zb = -0.4 if straddle else 0.3
    big = np.array([[(0, 0, 0.9, 1), (W, 0, 0.9, 1), (W, H, 0.9, 1)],
                    [(0, 0, 0.9, 1), (W, H, 0.9, 1), (0, H, zb, 1)],
                    [(-W, -H, 0.8, 1), (2 * W, H / 2, zb, 1), (W / 3, 2 * H, 0.6, 1)]], np.float32)
    col = np.array([[(1, 0, 0, 0), (0, 1, 0, 0), (0, 0, 1, 0)]] * 3, np.float32)
    return dataclasses.replace(sc, pos=np.concatenate([big, sc.pos]), col=np.concatenate([col, sc.col]))


@pytest.mark.parametrize("near", [False, True])
@pytest.mark.parametrize("model", ["kbk", "megakernel", "hybrid_rtc_mega", "hybrid_rtc_rtc"])
def test_raster_screen_filling_triangles_1080p(vpm, orc, model, near):
    """Triangles covering tens of thousands of 8x8 tiles at 1920x1080 (no VP_ERR_FANOUT),
    in both near-clip modes, bit-exact against the oracle."""
    from paper_conf_micro_zhengozsyc17_b200.workloads import RasterPipeline
    base = (inputs.raster_near_scene(n=2000, W=1920, H=1080, area_range=(0.5, 512.0)) if near
            else inputs.raster_scene(2000, W=1920, H=1080))
    scene = _with_big_triangles(base, near)
    rp = RasterPipeline(scene)
    configure(vpm, rp, model)
    ref = check(orc, scene, rp, rp.run())
    assert ref["n_fragment"] > 32_000   # the big triangles' tiles went through

"""Pins for the Reyes oracle (Fig. 1, L55).

Every check is anchored outside the oracle's own arithmetic: float64 Bezier/projection
math in numpy, a closed-form planar special case, the Kraft equality of a binary split
tree, conservation identities of the stage graph, and a brute-force per-pixel z-buffer
written here with an independent (perturbation) formulation of the fill rule.
"""
import math

import numpy as np
import pytest

from paper_conf_micro_zhengozsyc17_b200 import inputs

U64MAX = np.uint64(0xFFFFFFFFFFFFFFFF)


def bern64(t):
    return np.array([(1 - t) ** 3, 3 * t * (1 - t) ** 2, 3 * t * t * (1 - t), t ** 3])


def eval_patch64(cp, u, v):
    """float64 tensor-product Bezier: sum_a sum_b B_a(u) B_b(v) P[a][b]."""
    P = np.asarray(cp, np.float64).reshape(4, 4, 4)[:, :, :3]
    return np.einsum("a,b,abk->k", bern64(u), bern64(v), P)


def project64(M16, p3):
    M = np.asarray(M16, np.float64).reshape(4, 4)
    return M @ np.array([p3[0], p3[1], p3[2], 1.0])


# ------------------------------------------------------------------ elementary pieces
def test_project_matches_float64(orc):
    sc = inputs.reyes_config1()
    rng = np.random.default_rng(1)
    for _ in range(50):
        p = np.array([*rng.uniform(-1, 1, 3), 1.0], np.float32)
        c = orc.reyes_project(sc.M[0], p)
        ref = project64(sc.M[0], p[:3])
        assert np.allclose(c, ref, rtol=1e-5, atol=1e-5)


def test_shade_factor_special_cases(orc):
    L = np.array([0.0, 0.0, 1.0, 0.0], np.float32)
    assert orc.reyes_shade_factor([0, 0, 2], L) == pytest.approx(1.0, abs=1e-7)   # facing the light
    assert orc.reyes_shade_factor([0, 0, -2], L) == pytest.approx(0.1, abs=1e-7)  # facing away: ambient
    assert orc.reyes_shade_factor([0, 0, 0], L) == pytest.approx(0.1, abs=1e-7)   # degenerate normal
    L2 = inputs.default_light()
    n = np.array([0.3, -0.2, 0.9])
    ref = 0.1 + 0.9 * max(0.0, float(n @ L2[:3].astype(np.float64)) / np.linalg.norm(n))
    assert orc.reyes_shade_factor(n, L2) == pytest.approx(ref, abs=1e-6)


def test_split_halves_parameter_domain(orc):
    """de Casteljau at 1/2: child(t) == parent(t/2) (left) and parent((1+t)/2) (right)."""
    sc = inputs.reyes_config1()
    for k in (0, 5, 15):
        item = sc.seeds[k]
        for d in (0, 1):
            left, right = orc.reyes_split(item, d)
            for t in (0.0, 0.25, 0.5, 0.8, 1.0):
                for s in (0.0, 0.3, 1.0):
                    u, v = (t, s) if d == 0 else (s, t)
                    ul, vl = (t / 2, s) if d == 0 else (s, t / 2)
                    ur, vr = ((1 + t) / 2, s) if d == 0 else (s, (1 + t) / 2)
                    assert np.allclose(eval_patch64(left["cp"], u, v), eval_patch64(item["cp"], ul, vl), atol=1e-6)
                    assert np.allclose(eval_patch64(right["cp"], u, v), eval_patch64(item["cp"], ur, vr), atol=1e-6)
            assert left["depth"] == right["depth"] == item["depth"] + 1
            assert left["path"] == item["path"] and right["path"] == item["path"] | (1 << int(item["depth"]))
            assert (left["dirs"] >> int(item["depth"])) & 1 == d


def test_split_exact_on_dyadic_affine_patch(orc):
    sc = inputs.reyes_planar(48.0)
    left, right = orc.reyes_split(sc.seeds[0], 0)
    # x = a on the control grid -> left child x in {0, .5, 1, 1.5}, right {1.5, 2, 2.5, 3}
    assert left["cp"].reshape(4, 4, 4)[:, 0, 0].tolist() == [0.0, 0.5, 1.0, 1.5]
    assert right["cp"].reshape(4, 4, 4)[:, 0, 0].tolist() == [1.5, 2.0, 2.5, 3.0]


def test_dice_grid_matches_float64_bezier(orc):
    sc = inputs.reyes_config1()
    item = sc.seeds[6]
    g = orc.reyes_dice(sc, item)
    for i in range(9):
        for j in range(9):
            p = eval_patch64(item["cp"], i / 8, j / 8)
            k = i * 9 + j
            assert np.allclose(g[:3, k], p, atol=2e-6)
            c = project64(sc.M[0], p)
            assert g[3, k] == pytest.approx((c[0] / c[3] * 0.5 + 0.5) * sc.W, abs=2e-3)
            assert g[4, k] == pytest.approx((c[1] / c[3] * 0.5 + 0.5) * sc.H, abs=2e-3)
            assert g[5, k] == pytest.approx(c[2] / c[3], abs=1e-5)


def test_bound_classification_cases(orc):
    sc = inputs.reyes_planar(48.0, W=64, H=64)
    item = sc.seeds[0].copy()
    assert orc.reyes_bound(sc, item) == (orc.REYES_SPLIT, 0)   # 48 x 48 px > 8: split, tie -> u
    small = inputs.reyes_planar(6.0, W=64, H=64)
    assert orc.reyes_bound(small, small.seeds[0])[0] == orc.REYES_DICE
    off = inputs.reyes_planar(6.0, W=64, H=64, x0=70.0)
    assert orc.reyes_bound(off, off.seeds[0])[0] == orc.REYES_CULL   # bbox misses [0,W)
    wide = inputs.reyes_planar(48.0, W=64, H=64)
    wide.seeds["cp"][0, :, 1] *= 0.25                              # squash v: 48 x 12 px
    assert orc.reyes_bound(wide, wide.seeds[0]) == (orc.REYES_SPLIT, 0)
    tall = inputs.reyes_planar(48.0, W=64, H=64)
    tall.seeds["cp"][0, :, 0] *= 0.25                              # squash u: 12 x 48 px
    assert orc.reyes_bound(tall, tall.seeds[0]) == (orc.REYES_SPLIT, 1)
    behind = inputs.reyes_planar(48.0, W=64, H=64)
    behind.M = behind.M.copy()
    behind.M[0, 15] = -1.0                                         # every w = -1 <= near
    assert orc.reyes_bound(behind, behind.seeds[0])[0] == orc.REYES_CULL
    capped = inputs.reyes_planar(48.0, W=64, H=64)
    it = capped.seeds[0].copy()
    it["depth"] = 8
    assert orc.reyes_bound(capped, it)[0] == orc.REYES_DICE         # depth cap forces Dice


# ------------------------------------------------------------------ closed-form special case
@pytest.mark.parametrize("S,W,max_depth,leaves,depth", [
    (48.0, 64, 8, 64, 6),     # 48 -> 24x48 -> 24 -> 12x24 -> 12 -> 6x12 -> 6: 4^ceil(log2(48/8))
    (40.0, 64, 8, 64, 6),     # 4^ceil(log2 5) = 64
    (6.0, 64, 8, 1, 0),       # already diceable
    (200.0, 256, 4, 16, 4),   # 4^ceil(log2 25) = 1024, capped by depth 4 -> 4^2
])
def test_planar_patch_closed_form(orc, S, W, max_depth, leaves, depth):
    sc = inputs.reyes_planar(S, W=W, H=W, max_depth=max_depth)
    r = orc.reyes_definition(sc, leaf_cap=4096)
    assert r["n_dice"] == leaves and r["n_culled"] == 0
    assert r["depth_hist"][depth] == leaves
    # alternating u/v splits (tie -> u): n_split = leaves - 1
    assert r["n_split"] == leaves - 1
    # coverage: exactly the pixel centres inside [x0, x0+S)^2 (edges are off-centre)
    x0 = 8
    cov = r["key"][0] != U64MAX
    lo, hi = x0, int(math.floor(x0 + S - 0.5)) + 1
    exp = np.zeros((W, W), bool)
    exp[lo:hi, lo:hi] = True
    assert np.array_equal(cov, exp)
    # constant colour albedo * (0.1 + 0.9 * n.L) with n = +z, L = +z
    alb = sc.albedo[0, :3].astype(np.float64)
    col = r["colour"][0][cov]
    assert np.allclose(col[:, :3], alb * 1.0, atol=1e-6) and np.all(col[:, 3] == 1.0)
    assert np.all(r["colour"][0][~cov] == 0)


# ------------------------------------------------------------------ recursion invariants
def test_kraft_equality_per_patch(orc):
    """Leaves and culls of one patch partition its parameter domain:
    sum 2^-depth over leaves and culled nodes == 1 (exact in units of 2^-8)."""
    sc = inputs.reyes_config1()
    for k in range(sc.seeds.size):
        r = orc.reyes_definition(sc, seeds=sc.seeds[k:k + 1], leaf_cap=1024)
        total = sum(n << (8 - d) for d, n in enumerate(r["depth_hist"][:9]))
        total += sum(n << (8 - d) for d, n in enumerate(r["culled_depth_hist"][:9]))
        assert total == 256, (k, r["depth_hist"], r["culled_depth_hist"])
        assert sum(r["depth_hist"][9:]) == 0 and sum(r["culled_depth_hist"][9:]) == 0


def test_conservation_and_generator_selftest(orc):
    sc = inputs.reyes_config1()
    r = orc.reyes_definition(sc, leaf_cap=1 << 16)
    n_in = sc.seeds.size
    assert r["n_bound"] == n_in + 2 * r["n_split"]
    assert r["n_bound"] == r["n_split"] + r["n_dice"] + r["n_culled"]
    assert r["n_shade"] == r["n_dice"] == r["n_leaves"]
    # the config really exercises the depth cap and a dynamic range of depths
    assert r["depth_hist"][8] >= 1 and sum(r["depth_hist"][:5]) >= 1
    assert len(set(r["leaf_ids"].tolist())) == r["n_leaves"]


def test_definition_equals_pipeline(orc):
    for sc in (inputs.reyes_config1(), inputs.reyes_config5(n_frames=2, n_side=16)):
        a = orc.reyes_definition(sc, leaf_cap=1 << 17)
        b = orc.reyes_pipeline(sc, leaf_cap=1 << 17, trace_cap=1 << 19)
        for k in ("n_bound", "n_split", "n_dice", "n_shade", "n_culled", "depth_hist"):
            assert a[k] == b[k], k
        assert np.array_equal(a["key"], b["key"])
        assert np.array_equal(a["s"], b["s"])
        assert np.array_equal(a["colour"], b["colour"])
        assert sorted(a["leaf_ids"].tolist()) == sorted(b["leaf_ids"].tolist())
        tr = b["trace"]
        for st, n in zip(range(4), ("n_bound", "n_split", "n_dice", "n_shade")):
            ids = tr["id"][tr["stage"] == st]
            assert ids.size == b[n] and np.unique(ids).size == ids.size   # each (stage, id) once


# ------------------------------------------------------------------ brute force pixels
def _zkey(z32):
    b = np.float32(z32).view(np.uint32)
    return int(~b & 0xFFFFFFFF) if b & 0x80000000 else int(b | 0x80000000)


def _brute_force(sc, leaf_ids, grids):
    """Per pixel, min over every micropolygon of every leaf of (zkey << 32 | mp_id).
    Coverage via the perturbation form of the fill rule: sample at P - (e, e^2)."""
    W, H = sc.W, sc.H
    best = np.full((H, W), U64MAX, np.uint64)
    py, px = np.mgrid[0:H, 0:W]
    X = px.astype(np.int64) * 256 + 128
    Y = py.astype(np.int64) * 256 + 128
    for nid, g in zip(leaf_ids.tolist(), grids):
        patch = (nid >> 12) & 0xFFF
        depth = (nid >> 8) & 0xF
        path = nid & 0xFF
        for i in range(8):
            for j in range(8):
                ks = [i * 9 + j, (i + 1) * 9 + j, (i + 1) * 9 + j + 1, i * 9 + j + 1]  # v00 v10 v11 v01
                zq = (np.float32(g[5, ks[0]]) + np.float32(g[5, ks[1]])) + (np.float32(g[5, ks[2]]) + np.float32(g[5, ks[3]]))
                zq = np.float32(zq * np.float32(0.25))
                mp = (patch << 18) | (path << 10) | (depth << 6) | (i * 8 + j)
                key = np.uint64((_zkey(zq) << 32) | mp)
                V = [(int(np.rint(np.float64(g[3, k]) * 256)), int(np.rint(np.float64(g[4, k]) * 256))) for k in ks]
                for tri in ((V[0], V[1], V[2]), (V[0], V[2], V[3])):
                    (ax, ay), (bx, by), (cx, cy) = tri
                    area = (bx - ax) * (cy - ay) - (by - ay) * (cx - ax)
                    if area == 0:
                        continue
                    sgn = 1 if area > 0 else -1
                    inside = np.ones((H, W), bool)
                    for (x0, y0), (x1, y1) in (((ax, ay), (bx, by)), ((bx, by), (cx, cy)), ((cx, cy), (ax, ay))):
                        dx, dy = x1 - x0, y1 - y0
                        E = dx * (Y - y0) - dy * (X - x0)
                        tie = np.sign(dy) if dy != 0 else -np.sign(dx)   # E(P - (e,e^2)) = E + e*dy - e^2*dx
                        s = np.where(E != 0, np.sign(E), tie)
                        inside &= (s * sgn) > 0
                    upd = inside & (key < best)
                    best[upd] = key
    return best


@pytest.mark.parametrize("sl", [slice(0, 2), slice(12, 14), slice(5, 6)])
def test_brute_force_pixels_tiny(orc, sl):
    sc = inputs.reyes_config1(W=32, H=32)
    seeds = sc.seeds[sl]
    r = orc.reyes_definition(sc, seeds=seeds, leaf_cap=4096, want_grids=True)
    assert r["n_leaves"] > 0
    best = _brute_force(sc, r["leaf_ids"], r["leaf_grids"])
    assert np.array_equal(r["key"][0], best)
    # colour of every covered pixel = albedo[patch] * s of its winner
    cov = best != U64MAX
    patch = ((best[cov] >> np.uint64(18)) & np.uint64(0xFFF)).astype(np.int64)
    assert np.array_equal(r["colour"][0][cov][:, :3], sc.albedo[patch, :3] * r["s"][0][cov][:, None])


def test_brute_force_more_leaves(orc):
    """A 48x48 scene where near patches split several times."""
    sc = inputs.reyes_config1(W=48, H=48)
    seeds = sc.seeds[0:16:5]
    r = orc.reyes_definition(sc, seeds=seeds, leaf_cap=4096, want_grids=True)
    assert r["n_split"] > 0
    best = _brute_force(sc, r["leaf_ids"], r["leaf_grids"])
    assert np.array_equal(r["key"][0], best)


def test_planar_fill_rule_on_pixel_centres(orc):
    """Square edges through pixel centres (x0 = y0 = 8.5): sampling at P - (e, e^2)
    excludes the low edges and includes the high edges, so exactly px in [9, 9+S)."""
    S = 48.0
    sc = inputs.reyes_planar(S, W=64, H=64, x0=8.5, y0=8.5)
    r = orc.reyes_definition(sc, leaf_cap=4096)
    cov = r["key"][0] != U64MAX
    exp = np.zeros((64, 64), bool)
    exp[9:9 + int(S), 9:9 + int(S)] = True
    assert np.array_equal(cov, exp)


@pytest.mark.parametrize("S,x0,W,max_depth", [(48.0, 8.0, 64, 8), (40.0, 8.5, 64, 8), (6.0, 8.0, 64, 8),
                                               (200.0, 8.0, 256, 4), (48.0, 40.0, 64, 8)])
def test_planar_covering_micropolygon_count(orc, S, x0, W, max_depth):
    """The count of micropolygons whose (screen-clamped) box holds a pixel centre (what the
    GPU reports as Shade's work units) against a closed-form enumeration: the planar patch
    spans [x0, x0 + S]^2 px and is diced into a uniform (8 L) x (8 L) lattice of squares
    of side h = S / (8 L), L leaves per side; square k covers [x0 + k h, x0 + (k + 1) h] in
    x, and holds a column centre iff some integer c in [0, W) has c + 1/2 in that interval.
    The last case runs off the right / bottom edge (clamping)."""
    sc = inputs.reyes_planar(S, W=W, H=W, x0=x0, y0=x0, max_depth=max_depth)
    r = orc.reyes_definition(sc, leaf_cap=4096)
    d = [i for i, c in enumerate(r["depth_hist"]) if c]
    assert len(d) == 1 and d[0] % 2 == 0   # alternating u / v splits: every leaf at one depth
    per_side = 8 << (d[0] // 2)            # leaves wholly off screen are culled, and hold no centre
    h = S / per_side
    k = np.arange(per_side)
    lo, hi = x0 + k * h, x0 + (k + 1) * h
    has = np.array([any(a <= c + 0.5 <= b for c in range(W)) for a, b in zip(lo, hi)])
    assert r["n_mp_covering"] == int(has.sum()) ** 2
    assert orc.reyes_pipeline(sc)["n_mp_covering"] == r["n_mp_covering"]

"""Pins for the near-plane clipping mode of the rasterization oracle (
DESIGN.md reading R-S9).  Anchors independent of the oracle's clipping code:

- identity: with no vertex behind z = 0 the clip changes nothing but the id field
  (sub-id 2 tri), so the image equals the default mode's;
- orthographic equivalence: with w = 1 the default mode already discards fragments with
  z < 0 per pixel, and depth and colour are affine in screen space, so the clipped
  polygon covers the same pixels (up to the Q4 snap of the two new vertices) with the
  same depth and colour;
- sub-triangle counts by case (0, 1, 2, 3 vertices behind the plane);
- the definition and pipeline oracles agree bit for bit.
"""
import copy

import numpy as np
import pytest

from paper_conf_micro_zhengozsyc17_b200 import inputs

U64MAX = np.uint64(0xFFFFFFFFFFFFFFFF)
ID = np.uint64(0xFFFFFFFF)


def _z_of_key(k):
    b = (k >> np.uint64(32)).astype(np.uint32)
    return np.where(b & 0x80000000, b & 0x7FFFFFFF, ~b).astype(np.uint32).view(np.float32)


def _tri_scene(verts, W=64, H=64, near_clip=1):
    pos = np.zeros((1, 3, 4), np.float32)
    pos[0, :, :3] = np.asarray(verts, np.float32)
    pos[0, :, 3] = 1.0
    col = np.zeros((1, 3, 4), np.float32)
    col[0, :, :3] = np.eye(3, dtype=np.float32)
    return inputs.RasterScene(W=W, H=H, M=inputs.pixel_to_ndc(W, H), pos=pos, col=col, near_clip=near_clip)


def test_identity_without_vertices_behind(orc):
    sc = inputs.raster_scene(3000, W=160, H=120)
    a = orc.raster_definition(sc)
    sc2 = copy.deepcopy(sc)
    sc2.near_clip = 1
    b = orc.raster_definition(sc2)
    hit = a["key"] != U64MAX
    assert np.array_equal(hit, b["key"] != U64MAX)
    assert np.array_equal(a["key"][hit] >> np.uint64(32), b["key"][hit] >> np.uint64(32))
    assert np.array_equal((a["key"][hit] & ID) * np.uint64(2), b["key"][hit] & ID)
    assert np.array_equal(a["colour"], b["colour"])
    assert a["n_raster"] == b["n_raster"] and a["n_fragment"] == b["n_fragment"]


@pytest.mark.parametrize("seed", range(40))
def test_orthographic_equivalence_single_triangle(orc, seed):
    rng = np.random.default_rng(1000 + seed)
    v = np.zeros((3, 3))
    v[:, :2] = rng.uniform(4, 60, (3, 2))
    v[:, 2] = rng.uniform(-0.9, 0.9, 3)
    if (v[:, 2] >= 0).all() or (v[:, 2] < 0).all():
        v[0, 2], v[1, 2] = -abs(v[0, 2]) - 0.05, abs(v[1, 2]) + 0.05   # straddle
    a = orc.raster_definition(_tri_scene(v, near_clip=0))
    b = orc.raster_definition(_tri_scene(v, near_clip=1))
    ha, hb = a["key"] != U64MAX, b["key"] != U64MAX
    both = ha & hb
    # coverage differs only along the clip line / snapped new vertices: a thin band
    diff = int((ha ^ hb).sum())
    clip_len = 2 * 64  # generous bound: at most ~two pixel rows along a screen-long segment
    assert diff <= clip_len, (diff, int(ha.sum()), int(hb.sum()))
    assert int(hb.sum()) >= 0.8 * int(ha.sum()) - 4
    if both.any():
        # depth and colour are affine over the triangle: the only error is the Q4 snap of
        # the new vertices, levered across a possibly thin fan triangle; bound it by the
        # attribute's change over one pixel
        G = np.linalg.solve(np.c_[v[:, :2], np.ones(3)], np.c_[v[:, 2], np.eye(3)])[:2]
        gz, gc = np.abs(G[:, 0]).sum(), np.abs(G[:, 1:]).sum(0).max()
        za, zb = _z_of_key(a["key"][both]), _z_of_key(b["key"][both])
        assert np.max(np.abs(za - zb)) <= gz + 1e-5
        ca, cb = a["colour"][both], b["colour"][both]
        assert np.max(np.abs(ca - cb)) <= gc + 1e-4
    # every clipped-mode fragment is in front of the plane
    assert (_z_of_key(b["key"][hb]) >= 0).all()
    assert set(np.unique(b["key"][hb] & ID).tolist()) <= {0, 1}


@pytest.mark.parametrize("zs,n_sub", [((0.2, 0.3, 0.4), 1), ((-0.2, 0.3, 0.4), 2), ((-0.2, -0.3, 0.4), 1),
                                      ((-0.2, -0.3, -0.4), 0), ((0.0, 0.3, 0.4), 1), ((-0.2, 0.0, 0.4), 1),
                                      ((0.2, -0.3, 0.4), 2), ((0.2, 0.3, -0.4), 2), ((0.2, -0.3, -0.4), 1),
                                      ((-0.2, 0.3, -0.4), 1)])
def test_subtriangle_count_by_case(orc, zs, n_sub):
    v = [(8, 8, zs[0]), (56, 10, zs[1]), (30, 56, zs[2])]
    r = orc.raster_pipeline(_tri_scene(v))
    assert r["n_raster"] == n_sub
    assert r["n_clip"] == 1


def test_quad_split_covers_both_halves(orc):
    """One vertex behind: the 4-gon's two fan triangles (ids 0 and 1) both win pixels,
    and the colour at a pixel is the affine colour of the original triangle there."""
    v = [(4, 4, -0.5), (60, 4, 0.5), (32, 60, 0.5)]
    b = orc.raster_definition(_tri_scene(v))
    hb = b["key"] != U64MAX
    ids = b["key"][hb] & ID
    assert set(np.unique(ids).tolist()) == {0, 1}
    # the original triangle's barycentric colour (vertex colours = identity rows)
    X = np.array([p[0] for p in v], float)
    Y = np.array([p[1] for p in v], float)
    yy, xx = np.nonzero(hb)
    px, py = xx + 0.5, yy + 0.5
    A = (X[1] - X[0]) * (Y[2] - Y[0]) - (Y[1] - Y[0]) * (X[2] - X[0])
    l0 = ((X[2] - X[1]) * (py - Y[1]) - (Y[2] - Y[1]) * (px - X[1])) / A
    l1 = ((X[0] - X[2]) * (py - Y[2]) - (Y[0] - Y[2]) * (px - X[2])) / A
    l2 = 1 - l0 - l1
    want = np.stack([l0, l1, l2], 1)
    assert np.max(np.abs(b["colour"][hb][:, :3] - want)) <= 1e-3
    z = _z_of_key(b["key"][hb])
    assert np.max(np.abs(z - (-0.5 * l0 + 0.5 * l1 + 0.5 * l2))) <= 1e-3


def test_near_definition_equals_pipeline(orc):
    sc = inputs.raster_near_scene(3000, W=160, H=120)
    a = orc.raster_definition(sc)
    b = orc.raster_pipeline(sc, trace_cap=1 << 18)
    assert np.array_equal(a["key"], b["key"]) and np.array_equal(a["colour"], b["colour"])
    for k in ("n_vertex", "n_clip", "n_raster", "n_fragment", "n_frag_pixels"):
        assert a[k] == b[k], k
    assert sc.n_tris < b["n_raster"] <= 2 * sc.n_tris
    ids = b["trace"]["id"][b["trace"]["stage"] == 2]
    assert np.unique(ids).size == ids.size and (ids < 2 * sc.n_tris).all()


def test_perspective_clip_keeps_what_the_w_cull_drops(orc):
    """Perspective (w = z + 0.5): triangles with a vertex at w <= 0 are culled whole by
    the default mode; the clip keeps their front part, so it rasterises strictly more
    (sub-)triangles, and every pixel it shares with the default image at a triangle the
    default mode kept has the same depth within the snap bound."""
    sc = inputs.raster_near_scene(120, W=160, H=120, z_range=(-0.9, 0.95), perspective=True)
    b = orc.raster_definition(sc)
    sc0 = copy.deepcopy(sc)
    sc0.near_clip = 0
    a = orc.raster_definition(sc0)
    assert b["n_raster"] > a["n_raster"]
    assert int((b["key"] != U64MAX).sum()) > int((a["key"] != U64MAX).sum())
    assert (_z_of_key(b["key"][b["key"] != U64MAX]) >= 0).all()

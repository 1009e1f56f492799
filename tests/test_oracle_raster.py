"""Pins for the rasterization oracle (Fig. 16).

Anchors independent of the oracle's code: a pixel-major brute-force z-buffer written
here (no tiles, no stage decomposition), watertightness of a full-screen mesh, an exact
lattice-point count for a right triangle, and the stage-graph conservation identities.
"""
import numpy as np
import pytest

from paper_conf_micro_zhengozsyc17_b200 import inputs

U64MAX = np.uint64(0xFFFFFFFFFFFFFFFF)


def _zkey(z32):
    b = int(np.float32(z32).view(np.uint32))
    return (~b & 0xFFFFFFFF) if b & 0x80000000 else (b | 0x80000000)


def brute_force(scene):
    """Per pixel, argmin over all triangles of (zkey(z), tri); coverage by sampling at
    P - (e, e^2) (equivalent statement of the fill rule), float32 numpy arithmetic."""
    W, H = scene.W, scene.H
    best = np.full((H, W), U64MAX, np.uint64)
    M = scene.M.reshape(4, 4)
    f32 = np.float32
    for t in range(scene.n_tris):
        X, Y, Z = [], [], []
        clip = []
        for k in range(3):
            v = scene.pos[t, k]
            c = []
            for r in range(4):
                acc = f32(M[r, 0] * v[0])
                acc = f32(acc + f32(M[r, 1] * v[1]))
                acc = f32(acc + f32(M[r, 2] * v[2]))
                acc = f32(acc + f32(M[r, 3] * v[3]))
                c.append(acc)
            clip.append(c)
        outside = [all(c[0] < -c[3] for c in clip), all(c[0] > c[3] for c in clip), all(c[1] < -c[3] for c in clip),
                   all(c[1] > c[3] for c in clip), all(c[2] < 0 for c in clip), all(c[2] > c[3] for c in clip)]
        if any(outside):
            continue
        for c in clip:
            sx = f32(f32(f32(c[0] / c[3]) * f32(0.5)) + f32(0.5)) * f32(W)
            sy = f32(f32(f32(c[1] / c[3]) * f32(0.5)) + f32(0.5)) * f32(H)
            X.append(int(np.rint(f32(sx * f32(16)))))
            Y.append(int(np.rint(f32(sy * f32(16)))))
            Z.append(f32(c[2] / c[3]))
        area = (X[1] - X[0]) * (Y[2] - Y[0]) - (Y[1] - Y[0]) * (X[2] - X[0])
        if area == 0:
            continue
        if area < 0:
            X[1], X[2], Y[1], Y[2], Z[1], Z[2] = X[2], X[1], Y[2], Y[1], Z[2], Z[1]
            area = -area
        py, px = np.mgrid[0:H, 0:W]
        Px, Py = px.astype(np.int64) * 16 + 8, py.astype(np.int64) * 16 + 8
        E = []
        inside = np.ones((H, W), bool)
        for a, b in ((1, 2), (2, 0), (0, 1)):     # E_k opposite vertex k
            dx, dy = X[b] - X[a], Y[b] - Y[a]
            e = dx * (Py - Y[a]) - dy * (Px - X[a])
            tie = np.sign(dy) if dy != 0 else -np.sign(dx)
            inside &= np.where(e != 0, np.sign(e), tie) > 0
            E.append(e)
        for yy, xx in zip(*np.nonzero(inside)):
            l = [f32(f32(E[k][yy, xx]) / f32(area)) for k in range(3)]
            z = f32(f32(l[0] * Z[0]) + f32(l[1] * Z[1]))
            z = f32(z + f32(l[2] * Z[2]))
            if not (0.0 <= z <= 1.0):
                continue
            key = np.uint64((_zkey(z) << 32) | t)
            if key < best[yy, xx]:
                best[yy, xx] = key
    return best


@pytest.mark.parametrize("seed", [1, 2])
def test_brute_force_tiny(orc, seed):
    sc = inputs.raster_scene(200, W=64, H=64, seed=inputs.seed_for(4, seed), area_range=(0.5, 200.0))
    r = orc.raster_pipeline(sc)
    assert np.array_equal(r["key"], brute_force(sc))


def test_definition_equals_pipeline(orc):
    sc = inputs.raster_scene(20000, W=320, H=180)
    a = orc.raster_definition(sc)
    b = orc.raster_pipeline(sc, trace_cap=1 << 20)
    assert np.array_equal(a["key"], b["key"]) and np.array_equal(a["colour"], b["colour"])
    for k in ("n_vertex", "n_clip", "n_raster", "n_fragment", "n_frag_pixels"):
        assert a[k] == b[k], k
    # conservation (SURVEY c-5 pin 4)
    assert b["n_vertex"] == b["n_clip"] == sc.n_tris
    assert b["n_raster"] <= sc.n_tris and b["n_fragment"] >= b["n_raster"]
    tr = b["trace"]
    for st, n in enumerate(("n_vertex", "n_clip", "n_raster", "n_fragment")):
        ids = tr["id"][tr["stage"] == st]
        assert ids.size == b[n] and np.unique(ids).size == ids.size


def test_watertight_quad_mesh(orc):
    """A full-screen mesh covers every pixel centre exactly once (fragments = W*H)."""
    sc = inputs.raster_quad_mesh(64, 48, cell=8)
    r = orc.raster_pipeline(sc)
    assert r["n_frag_pixels"] == 64 * 48
    assert np.all(r["key"] != U64MAX)
    assert np.allclose(r["colour"][..., :3], 0.5, atol=1e-6) and np.all(r["colour"][..., 3] == 1)


@pytest.mark.parametrize("a,b", [(10, 7), (13, 5), (3, 17), (6, 6)])
def test_right_triangle_lattice_count(orc, a, b):
    """Legs of a and b pixels from the pixel corner (x0, y0): covered centres are the
    (i, j) >= 0 with (2i+1)/a + (2j+1)/b < 2, plus the centres ON the hypotenuse: it runs
    v1 -> v2 with dy > 0, so the fill rule gives it its boundary (legs carry no centres)."""
    x0, y0 = 5, 6
    sc = inputs.raster_scene(1, W=64, H=64)
    sc.pos[0, :, 0] = [x0, x0 + a, x0]
    sc.pos[0, :, 1] = [y0, y0, y0 + b]
    sc.pos[0, :, 2] = 0.5
    exp = sum(1 for i in range(a) for j in range(b) if (2 * i + 1) * b + (2 * j + 1) * a < 2 * a * b)
    ties = sum(1 for i in range(a) for j in range(b) if (2 * i + 1) * b + (2 * j + 1) * a == 2 * a * b)
    exp += ties
    r = orc.raster_pipeline(sc)
    assert r["n_frag_pixels"] == exp
    cov = r["key"] != U64MAX
    assert cov.sum() == exp and cov[y0:y0 + b, x0:x0 + a].sum() == exp


def test_barycentric_colour_interpolation(orc):
    """Constant-colour triangle resolves to that colour; z-buffer keeps the nearer one."""
    sc = inputs.raster_scene(2, W=64, H=64)
    for t, z in ((0, 0.7), (1, 0.3)):
        sc.pos[t, :, 0] = [4, 60, 4]
        sc.pos[t, :, 1] = [4, 4, 60]
        sc.pos[t, :, 2] = z
        sc.col[t, :, :3] = [0.25 * (t + 1), 0.5, 0.125]
    r = orc.raster_pipeline(sc)
    cov = r["key"] != U64MAX
    assert np.all((r["key"][cov] & np.uint64(0xFFFFFFFF)) == 1)      # the nearer triangle wins
    assert np.allclose(r["colour"][cov][:, :3], [0.5, 0.5, 0.125], atol=1e-6)

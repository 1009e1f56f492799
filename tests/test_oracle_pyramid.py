"""Pins for the image-pyramid oracle (Fig. 12).

Independent anchors: the Wikipedia histogram-equalisation worked example (golden file),
a numpy re-derivation of the whole pyramid written here, closed-form level sizes and
task counts, constant-image and LUT invariants.
"""
import json
import os

import numpy as np
import pytest

from paper_conf_micro_zhengozsyc17_b200 import inputs

GOLDEN = os.path.join(os.path.dirname(__file__), "golden")


def test_histeq_wikipedia_example(orc):
    g = json.load(open(os.path.join(GOLDEN, "histeq_wikipedia.json")))
    img = np.array(g["image"], np.int64)
    hist = np.bincount(img.ravel(), minlength=256)
    lut = orc.histeq_lut(hist, img.size)
    assert np.array_equal(lut[img], np.array(g["equalized"]))


def test_histeq_invariants(orc):
    rng = np.random.default_rng(0)
    for _ in range(20):
        vals = rng.integers(0, 256, size=rng.integers(2, 2000))
        hist = np.bincount(vals, minlength=256)
        lut = orc.histeq_lut(hist, vals.size).astype(int)
        nz = np.nonzero(hist)[0]
        assert np.all(np.diff(lut) >= 0)
        assert lut[nz[0]] == 0
        if nz.size > 1:
            assert lut[nz[-1]] == 255
    # constant image: N == cmin -> identity
    assert np.array_equal(orc.histeq_lut(np.bincount([7] * 50, minlength=256), 50), np.arange(256))


def numpy_pyramid(rgb):
    """Textbook re-derivation with whole-array numpy ops."""
    r, g, b = (rgb[..., k].astype(np.int64) for k in range(3))
    gray = (77 * r + 150 * g + 29 * b + 128) >> 8
    out = []
    for i in range(rgb.shape[0]):
        gi = gray[i]
        hist = np.bincount(gi.ravel(), minlength=256)
        cdf = np.cumsum(hist)
        N = gi.size
        first = np.nonzero(hist)[0][0]
        cmin = cdf[first]
        if N == cmin:
            lut = np.arange(256)
        else:
            lut = np.where(np.arange(256) < first, 0, ((cdf - cmin) * 255 + (N - cmin) // 2) // (N - cmin))
        lev = lut[gi]
        levels = [lev]
        while lev.shape[0] > 1:
            lev = (lev[0::2, 0::2] + lev[0::2, 1::2] + lev[1::2, 0::2] + lev[1::2, 1::2] + 2) >> 2
            levels.append(lev)
        out.append(np.concatenate([l.ravel() for l in levels]).astype(np.uint8))
    return np.stack(out)


def resize_count(S, T=64):
    """Closed form: level l >= 1 has max(1, (S>>l)/T)^2 output tiles."""
    n, l = 0, 1
    while (S >> l) >= 1:
        t = max(1, (S >> l) // T)
        n += t * t
        l += 1
    return n


@pytest.mark.parametrize("S,n", [(256, 2), (512, 2), (64, 3)])
def test_pyramid_matches_numpy_and_counts(orc, S, n):
    rgb = inputs.pyramid_images(n, S)
    d = orc.pyr_definition(rgb)
    p = orc.pyr_pipeline(rgb, trace_cap=1 << 16)
    ref = numpy_pyramid(rgb)
    assert np.array_equal(d["pyr"], ref) and np.array_equal(p["pyr"], ref)
    assert d["levels"] == int(np.log2(S)) + 1
    assert orc.pyr_level_offset(S, d["levels"]) == sum((S >> l) ** 2 for l in range(d["levels"]))
    t0 = (S // 64) ** 2
    assert p["n_gray"] == n * t0 and p["n_cdf"] == n
    assert p["n_map"] == n * (S // 64) * -(-(S // 64) // 8)
    assert p["n_resize"] == n * resize_count(S)
    tr = p["trace"]
    for st, k in enumerate(("n_gray", "n_cdf", "n_map", "n_resize")):
        ids = tr["id"][tr["stage"] == st]
        assert ids.size == p[k] and np.unique(ids).size == ids.size


def test_resize_count_full_size():
    # 1 371 Resize latches per 4096^2 image (1024+256+64+16+4+7x1)
    assert resize_count(4096) == 1371


def test_constant_image_constant_pyramid(orc):
    rgb = np.full((1, 128, 128, 3), 90, np.uint8)
    p = orc.pyr_pipeline(rgb)
    y = (77 * 90 + 150 * 90 + 29 * 90 + 128) >> 8
    assert np.all(p["pyr"] == y)          # LUT = identity, box filter keeps constants


def test_grayscale_weights_against_bt601(orc):
    """Reading R-P1's integer weights (77, 150, 29)/256 against ITU-R BT.601 luma in float64,
    Y = 0.299 R + 0.587 G + 0.114 B: the oracle's level-0 gray image is within one grey level
    of round(Y) for every (R, G) pair and 64 blue values (4 Mi colours, the extremes
    included), and exact on the neutral axis R = G = B (where Y = R)."""
    r, g = np.meshgrid(np.arange(256), np.arange(256), indexing="ij")
    blues = np.unique(np.concatenate([np.linspace(0, 255, 63).astype(int), [128]]))
    assert blues.size == 64 and blues[0] == 0 and blues[-1] == 255
    rgb = np.zeros((2048, 2048, 3), np.uint8)
    tiles = rgb.reshape(8, 256, 8, 256, 3)
    for k, b in enumerate(blues):
        t = tiles[k // 8, :, k % 8, :, :]
        t[..., 0], t[..., 1], t[..., 2] = r, g, b
    res = orc.pyr_definition(rgb[None])
    gray = res["gray"][0].reshape(2048, 2048).astype(np.int64)
    y = np.rint(0.299 * rgb[..., 0] + 0.587 * rgb[..., 1] + 0.114 * rgb[..., 2]).astype(np.int64)
    assert np.max(np.abs(gray - y)) <= 1
    neutral = (rgb[..., 0] == rgb[..., 1]) & (rgb[..., 1] == rgb[..., 2])
    assert neutral.sum() >= 64 and np.array_equal(gray[neutral], rgb[..., 0][neutral].astype(np.int64))

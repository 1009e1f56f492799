"""Pins for the LBP face-detection oracle (Fig. 14).

Independent anchors: the level sizes and the 5 306 934-window count of a 1920x1080 frame
(closed forms), a vectorised numpy re-derivation of gray/HistEq/resize/LBP/cascade over
every window, constant-image invariants, and the planted templates being detected."""
import numpy as np
import pytest

from paper_conf_micro_zhengozsyc17_b200 import inputs

LEVELS_1080P = [(1920, 1080), (1536, 864), (1228, 691), (982, 552), (785, 441), (628, 352), (502, 281), (401, 224)]


def test_level_sizes_and_window_count(orc):
    lv = orc.fd_levels(1920, 1080)
    assert lv == LEVELS_1080P
    assert sum((w - 23) * (h - 23) for w, h in lv) == 5_306_934      # SURVEY §8(c-2) pin 6
    assert orc.fd_levels(30, 30) == [(30, 30), (24, 24)] and orc.fd_levels(29, 40) == [(29, 40)]


def numpy_facedet(sc):
    """Whole-array re-derivation (per frame): levels, LBP, survivors, detections."""
    dets, surv = [], np.zeros(len(sc.n_weak), np.int64)
    for f in range(sc.n_frames):
        rgb = sc.rgb[f].astype(np.int64)
        gray = (77 * rgb[..., 0] + 150 * rgb[..., 1] + 29 * rgb[..., 2] + 128) >> 8
        hist = np.bincount(gray.ravel(), minlength=256)
        cdf = np.cumsum(hist)
        N, first = gray.size, np.nonzero(hist)[0][0]
        cmin = cdf[first]
        lut = np.arange(256) if N == cmin else np.where(np.arange(256) < first, 0,
                                                        ((cdf - cmin) * 255 + (N - cmin) // 2) // (N - cmin))
        img = lut[gray]
        w, h = sc.W, sc.H
        level = 0
        while level < 8 and w >= 24 and h >= 24:
            if level > 0:
                nw, nh = (4 * w) // 5, (4 * h) // 5
                if nw < 24 or nh < 24:
                    break
                img = img[(5 * np.arange(nh)) >> 2][:, (5 * np.arange(nw)) >> 2]
                w, h = nw, nh
            lbp = np.zeros((h, w), np.int64)
            c = img[1:-1, 1:-1]
            for p, (dx, dy) in enumerate([(-1, -1), (0, -1), (1, -1), (1, 0), (1, 1), (0, 1), (-1, 1), (-1, 0)]):
                nbv = img[1 + dy:h - 1 + dy, 1 + dx:w - 1 + dx]
                lbp[1:-1, 1:-1] |= (nbv >= c).astype(np.int64) << p
            ys, xs = np.mgrid[0:h - 23, 0:w - 23]
            alive = np.ones(ys.shape, bool)
            wi = 0
            for k, nk in enumerate(sc.n_weak):
                s = np.zeros(ys.shape, np.int64)
                for _ in range(nk):
                    cx, cy = sc.weak[wi, 0], sc.weak[wi, 1]
                    masks = sc.weak[wi, 2:10].astype(np.uint32)
                    code = lbp[ys + cy, xs + cx]
                    bit = (masks[code >> 5] >> (code & 31).astype(np.uint32)) & 1
                    s += np.where(bit == 1, sc.weak[wi, 10], sc.weak[wi, 11])
                    wi += 1
                alive &= s >= sc.thr[k]
                surv[k] += alive.sum()
            for y, x in zip(*np.nonzero(alive)):
                dets.append((f, level, x, y))
            level += 1
    return sorted(dets), surv.tolist()


@pytest.mark.parametrize("W,H,F", [(480, 270, 1), (200, 120, 2)])
def test_matches_numpy_rederivation(orc, W, H, F):
    sc = inputs.face_scene(W=W, H=H, n_frames=F, n_planted=4)
    a = orc.fd_definition(sc)
    b = orc.fd_pipeline(sc, trace_cap=1 << 20)
    dets, surv = numpy_facedet(sc)
    for r in (a, b):
        assert sorted(map(tuple, r["det"].tolist())) == dets
        assert r["survivors"] == surv
    assert np.array_equal(a["levels"], b["levels"]) and np.array_equal(a["lbp"], b["lbp"])
    assert a["windows"] == b["windows"] == F * sum((w - 23) * (h - 23) for w, h in orc.fd_levels(W, H))
    # stage counts: Gray/Map per band, CDF per frame, Resize/LBP per (level, band), Scan per window row
    lv = orc.fd_levels(W, H)
    bands = [-(-h // 32) for _, h in lv]
    assert b["deq"] == [F * bands[0], F, F * bands[0], F * sum(bands[1:]), F * sum(bands),
                        F * sum(h - 23 for _, h in lv)]
    tr = b["trace"]
    for st in range(6):
        ids = tr["id"][tr["stage"] == st]
        assert ids.size == b["deq"][st] and np.unique(ids).size == ids.size


def test_planted_templates_detected_and_constant_invariants(orc):
    sc = inputs.face_scene(W=320, H=200, n_planted=6)
    r = orc.fd_pipeline(sc)
    found = {(int(x), int(y)) for f, l, x, y in r["det"].tolist() if l == 0}
    for x, y in sc.planted[0].tolist():
        assert (x, y) in found
    assert r["survivors"][-1] == r["n_det"]
    const = inputs.face_scene(W=64, H=48, n_planted=0)
    const.rgb[:] = 77
    rc = orc.fd_definition(const)
    assert np.array_equal(rc["lut"][0], np.arange(256))                 # N == cmin: identity
    lb = rc["lbp"][0][: 64 * 48].reshape(48, 64)
    assert np.all(lb[1:-1, 1:-1] == 255) and lb[0].sum() == lb[-1].sum() == 0


def test_grayscale_bins_against_bt601(orc):
    """Face detection's own grayscale (oracle/facedet.c, reading R-D1) against float64
    BT.601 luma: a constant frame of colour c puts all its pixels into one histogram bin,
    which must be within one grey level of round(0.299 R + 0.587 G + 0.114 B)."""
    from paper_conf_micro_zhengozsyc17_b200 import inputs
    base = inputs.face_scene(W=24, H=24, n_frames=1, n_planted=0)
    rng = np.random.default_rng(601)
    cols = np.concatenate([rng.integers(0, 256, (250, 3)), [[0, 0, 0], [255, 255, 255], [255, 0, 0], [0, 255, 0],
                                                            [0, 0, 255], [128, 128, 128]]]).astype(np.uint8)
    rgb = np.broadcast_to(cols[:, None, None, :], (cols.shape[0], 24, 24, 3)).copy()
    sc = inputs.FaceScene(W=24, H=24, rgb=rgb, n_weak=base.n_weak, thr=base.thr, weak=base.weak,
                          planted=np.zeros((cols.shape[0], 0, 2), np.int32))
    res = orc.fd_definition(sc)
    for f, c in enumerate(cols.astype(np.float64)):
        nz = np.nonzero(res["hist"][f])[0]
        assert nz.size == 1 and res["hist"][f][nz[0]] == 24 * 24
        assert abs(int(nz[0]) - int(np.rint(0.299 * c[0] + 0.587 * c[1] + 0.114 * c[2]))) <= 1, (c, nz[0])

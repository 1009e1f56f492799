"""Host-side checks of the 208-B queued Reyes patch item (reading R-S10): the
repack of the paper's 272-B item keeps every control-point coordinate and header field,
the generators only ever produce affine control points (w == 1), and a w != 1 seed is
rejected instead of being silently flattened."""
import numpy as np
import pytest

from paper_conf_micro_zhengozsyc17_b200 import inputs


def test_gpu_patch_item_layout():
    assert inputs.PATCH_DTYPE.itemsize == 272
    assert inputs.GPU_PATCH_DTYPE.itemsize == 208
    # x, y, z planes first (16-B aligned rows for the Dice loads), then the header
    offs = {n: inputs.GPU_PATCH_DTYPE.fields[n][1] for n in inputs.GPU_PATCH_DTYPE.names}
    assert offs == {"x": 0, "y": 64, "z": 128, "id": 192, "path": 196, "dirs": 200, "depth": 204}


@pytest.mark.parametrize("make", [lambda: inputs.reyes_config1(), lambda: inputs.reyes_config5(n_frames=2)])
def test_gpu_patch_items_repack(make):
    sc = make()
    assert np.all(sc.seeds["cp"][..., 3] == np.float32(1.0))    # affine control points
    g = inputs.gpu_patch_items(sc.seeds)
    assert g.shape == sc.seeds.shape
    for c, name in enumerate("xyz"):
        assert np.array_equal(g[name].view(np.uint32), sc.seeds["cp"][..., c].view(np.uint32))
    for name in ("id", "path", "dirs", "depth"):
        assert np.array_equal(g[name], sc.seeds[name])
    # raw bytes: point k of plane c sits at 64 c + 4 k
    raw = g.view(np.uint8).reshape(g.size, 208)
    k = 7
    assert raw[0, 64 + 4 * k:68 + 4 * k].view(np.float32)[0] == sc.seeds["cp"][0, k, 1]


def test_gpu_patch_items_rejects_projective_points():
    sc = inputs.reyes_config1()
    s = sc.seeds.copy()
    s["cp"][3, 5, 3] = np.float32(2.0)
    with pytest.raises(ValueError):
        inputs.gpu_patch_items(s)
    assert inputs.gpu_patch_items(s[:0]).size == 0

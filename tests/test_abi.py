"""CPU-side checks of the boundary: libvp.so builds, loads without a GPU, and exports
every entry point include/vp.h declares; struct layouts of the binding match the header."""
import ctypes
import os
import re
import subprocess

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
HDR = os.path.join(ROOT, "include", "vp.h")


def declared_functions():
    src = open(HDR).read()
    src = re.sub(r"/\*.*?\*/", "", src, flags=re.S)
    return sorted(set(re.findall(r"^\s*(?:vp_status|const char\*)\s+(vp_\w+)\s*\(", src, flags=re.M)))


@pytest.fixture(scope="module")
def lib():
    from paper_conf_micro_zhengozsyc17_b200 import build
    path = build.build()
    return ctypes.CDLL(path)


def test_every_declared_symbol_is_exported(lib):
    fns = declared_functions()
    assert len(fns) >= 15
    for f in fns:
        assert hasattr(lib, f), f"libvp.so does not export {f}"


def test_exports_are_extern_c():
    from paper_conf_micro_zhengozsyc17_b200 import build
    out = subprocess.run(["nm", "-D", "--defined-only", build.build()], capture_output=True, text=True).stdout
    exported = set(re.findall(r"\bT (vp_\w+)", out))
    assert set(declared_functions()) <= exported


def test_binding_declares_all_symbols():
    from paper_conf_micro_zhengozsyc17_b200 import vp
    assert set(declared_functions()) == set(vp.EXPORTED)


def test_struct_sizes_match_header():
    """Compile a tiny C program against vp.h and compare sizeof with the ctypes mirrors."""
    from paper_conf_micro_zhengozsyc17_b200 import vp
    prog = r'''
#include <stdio.h>
#include "vp.h"
int main(void){printf("%zu %zu %zu %zu %zu %zu %zu %zu %zu %zu %zu %zu %zu %zu %zu\n", sizeof(vp_pipeline_desc), sizeof(vp_stage_desc),
 sizeof(vp_sm_binding), sizeof(vp_config), sizeof(vp_run_stats), sizeof(vp_autotune_opts), sizeof(vp_tune_report),
 sizeof(vp_toy_params), sizeof(vp_collatz_params), sizeof(vp_reyes_params), sizeof(vp_raster_params),
 sizeof(vp_pyramid_params), sizeof(vp_cfd_params), sizeof(vp_facedet_params), sizeof(vp_qbench_params));return 0;}
'''
    tmp = os.path.join(ROOT, "build_abi_check")
    os.makedirs(tmp, exist_ok=True)
    c = os.path.join(tmp, "sz.c")
    open(c, "w").write(prog)
    exe = os.path.join(tmp, "sz")
    subprocess.run(["gcc", "-I", os.path.join(ROOT, "include"), c, "-o", exe], check=True)
    sizes = [int(x) for x in subprocess.run([exe], capture_output=True, text=True).stdout.split()]
    mirrors = [vp.PipelineDesc, vp.StageDesc, vp.SmBinding, vp.Config, vp.RunStats, vp.AutotuneOpts, vp.TuneReport,
               vp.ToyParams, vp.CollatzParams, vp.ReyesParams, vp.RasterParams, vp.PyramidParams, vp.CfdParams,
               vp.FaceDetParams, vp.QBenchParams]
    assert sizes == [ctypes.sizeof(m) for m in mirrors]


def test_no_gpu_calls_fail_cleanly(lib):
    """Without a GPU the library reports an error instead of crashing."""
    import torch
    if torch.cuda.is_available():
        pytest.skip("GPU present")
    from paper_conf_micro_zhengozsyc17_b200 import vp
    with pytest.raises(vp.VPError):
        vp.Pipeline(0)


def test_config_string_roundtrip():
    """vp_config_to_string / vp_config_from_string are host-only (no GPU needed)."""
    from paper_conf_micro_zhengozsyc17_b200 import vp
    b = vp.make_binding([(0, 1, vp.GROUP_MEGA, 0, 44), (2, 3, vp.GROUP_RTC, 44, 148)], 148,
                        blocks_per_sm=[2, 0, 3, 0], batch=[32, 16, 8, 4])
    c = vp.Config(model=vp.HYBRID, has_binding=1, binding=b, batch=0)
    g = vp.Config(model=vp.KBK_GRAPH, has_binding=0, batch=0)
    assert vp.config_from_string(vp.config_to_string(g)).model == vp.KBK_GRAPH
    s = vp.config_to_string(c)
    c2 = vp.config_from_string(s)
    assert ctypes.string_at(ctypes.addressof(c), ctypes.sizeof(c)) == ctypes.string_at(ctypes.addressof(c2), ctypes.sizeof(c2))
    assert vp.config_to_string(c2) == s
    with pytest.raises(vp.VPError):
        vp.config_from_string("garbage")


def test_stage_kind_info_host_only():
    """vp_stage_kind_info needs no device: the strides every built-in kind is registered with
    (include/vp.h: 208-B patches for Reyes Bound/Split/Dice, reading R-S10; 1968-B grids)."""
    from paper_conf_micro_zhengozsyc17_b200 import vp
    assert [vp.stage_kind_info(k)[0] for k in (vp.REYES_BOUND, vp.REYES_SPLIT, vp.REYES_DICE, vp.REYES_SHADE)] == [
        208, 208, 208, 2032]
    assert [vp.stage_kind_info(k)[1] for k in (vp.REYES_BOUND, vp.REYES_SPLIT, vp.REYES_DICE, vp.REYES_SHADE)] == [
        16, 16, 32, 64]
    assert vp.stage_kind_info(vp.TOY_S1) == (4, 1)
    # queue microbenchmark: plain and cluster-stealing kinds share their item layouts
    assert [vp.stage_kind_info(k)[0] for k in (vp.QB_ITEM4, vp.QB_ITEM16, vp.QB_ITEM272, vp.QB_ITEM4_CS,
                                                vp.QB_ITEM16_CS)] == [4, 16, 272, 4, 16]
    with pytest.raises(vp.VPError):
        vp.stage_kind_info(9999)

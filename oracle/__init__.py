"""CPU ORACLE — test infrastructure only.

ctypes wrapper around ``oracle/liboracle.so`` (plain C, see ``oracle/oracle.h``).  Only
``tests/``, ``__graft_entry__.smoke()`` and ``bench.py``'s cpu_baseline / ``--impl
reference`` leg may import this module.  It never imports the CUDA path; inputs arrive
as plain numpy arrays (or any object with the ReyesScene attributes) produced by
``paper_conf_micro_zhengozsyc17_b200/inputs.py``.
"""
from __future__ import annotations

import ctypes as C
import os
import subprocess

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_LIB_PATH = os.path.join(_HERE, "liboracle.so")


def build(force: bool = False) -> str:
    """Compile the C oracle (make -C oracle)."""
    if force or not os.path.exists(_LIB_PATH) or any(
            os.path.getmtime(os.path.join(_HERE, f)) > os.path.getmtime(_LIB_PATH)
            for f in os.listdir(_HERE) if f.endswith((".c", ".h"))):
        subprocess.run(["make", "-s", "-C", _HERE], check=True)
    return _LIB_PATH


_lib = None


def lib():
    global _lib
    if _lib is None:
        build()
        _lib = C.CDLL(_LIB_PATH)
        _declare(_lib)
    return _lib


MAX_STAGES = 8
P = C.c_void_p


class Stats(C.Structure):
    _fields_ = [("deq", C.c_uint64 * MAX_STAGES), ("enq", C.c_uint64 * MAX_STAGES)]


class TraceRec(C.Structure):
    _fields_ = [("id", C.c_uint64), ("stage", C.c_uint32), ("pad", C.c_uint32)]


TRACE_DTYPE = np.dtype([("id", "<u8"), ("stage", "<u4"), ("pad", "<u4")])


class ReyesSceneC(C.Structure):
    _fields_ = [("W", C.c_int32), ("H", C.c_int32), ("n_frames", C.c_int32),
                ("patches_per_frame", C.c_int32), ("max_depth", C.c_int32), ("pad0", C.c_int32),
                ("t_dice", C.c_float), ("near_w", C.c_float), ("M", P), ("albedo", P),
                ("L", C.c_float * 4)]


class ReyesOutC(C.Structure):
    _fields_ = [("key", P), ("s", P), ("colour", P),
                ("n_bound", C.c_uint64), ("n_split", C.c_uint64), ("n_dice", C.c_uint64),
                ("n_shade", C.c_uint64), ("n_culled", C.c_uint64),
                ("depth_hist", C.c_uint64 * 16), ("culled_depth_hist", C.c_uint64 * 16),
                ("leaf_ids", P), ("leaf_cap", C.c_size_t), ("n_leaves", C.c_size_t),
                ("leaf_grids", P),
                ("trace", P), ("trace_cap", C.c_size_t), ("trace_n", C.c_size_t),
                ("n_mp_covering", C.c_uint64)]


def _declare(L):
    L.orc_toy_definition.argtypes = [P, C.c_size_t, C.c_int32, P, P]
    L.orc_toy_pipeline.argtypes = [P, C.c_size_t, C.c_int32, P, P, P]
    L.orc_qbench_pipeline.argtypes = [P, C.c_size_t, C.c_size_t, C.c_uint32, P, P, P, P]
    L.orc_ldpc_definition.argtypes = [P, P, P]
    L.orc_ldpc_pipeline.argtypes = [P, P, P, P]
    L.orc_collatz_definition.argtypes = [P, C.c_size_t, P]
    L.orc_collatz_pipeline.argtypes = [P, C.c_size_t, C.c_uint32, P, P, P]
    L.orc_reyes_definition.argtypes = [P, P, C.c_size_t, P]
    L.orc_reyes_pipeline.argtypes = [P, P, C.c_size_t, P]
    L.orc_reyes_bound.argtypes = [P, P, P]
    L.orc_reyes_split.argtypes = [P, C.c_int, P, P]
    L.orc_reyes_dice.argtypes = [P, P, P]
    L.orc_reyes_project.argtypes = [P, P, P]
    L.orc_reyes_shade_factor.argtypes = [P, P]
    L.orc_reyes_shade_factor.restype = C.c_float


def _ptr(a: np.ndarray):
    assert a.flags["C_CONTIGUOUS"]
    return a.ctypes.data_as(C.c_void_p)


# ------------------------------------------------------------------ toy / collatz
def toy_definition(seeds: np.ndarray, threshold: int):
    seeds = np.ascontiguousarray(seeds, np.int32)
    out = np.zeros_like(seeds)
    passes = C.c_uint64(0)
    rc = lib().orc_toy_definition(_ptr(seeds), seeds.size, threshold, _ptr(out), C.byref(passes))
    assert rc == 0
    return out, passes.value


def toy_pipeline(seeds: np.ndarray, threshold: int):
    seeds = np.ascontiguousarray(seeds, np.int32)
    out = np.zeros_like(seeds)
    n_out = C.c_size_t(0)
    st = Stats()
    rc = lib().orc_toy_pipeline(_ptr(seeds), seeds.size, threshold, _ptr(out), C.byref(n_out), C.byref(st))
    assert rc == 0
    return out[: n_out.value], list(st.deq[:3]), list(st.enq[:3])


def qbench_pipeline(seeds: np.ndarray, item_bytes: int, fanout: int):
    """Queue microbenchmark (qbench.c): returns (leaves, id sum, bad payloads, tasks dequeued)."""
    seeds = np.ascontiguousarray(seeds, np.uint32)
    assert seeds.size * 4 % item_bytes == 0
    n = seeds.size * 4 // item_bytes
    lv, ids, bad = C.c_uint64(0), C.c_uint64(0), C.c_uint64(0)
    st = Stats()
    rc = lib().orc_qbench_pipeline(_ptr(seeds), n, item_bytes, fanout, C.byref(lv), C.byref(ids), C.byref(bad),
                                   C.byref(st))
    assert rc == 0
    return lv.value, ids.value, bad.value, int(st.deq[0])


class LdpcC(C.Structure):
    _fields_ = [("N", C.c_int32), ("M", C.c_int32), ("dv", C.c_int32), ("dc", C.c_int32), ("n_frames", C.c_int32),
                ("n_iter", C.c_int32), ("alpha", C.c_float), ("nc_chk", C.c_int32), ("nc_var", C.c_int32),
                ("pad", C.c_int32), ("check_vars", P), ("var_edges", P), ("llr", P)]


def _ldpc_run(fn, sc, llr=None, n_iter=None, alpha=None):
    llr = np.ascontiguousarray(sc.llr if llr is None else llr, np.float32)
    cv = np.ascontiguousarray(sc.check_vars, np.int32)
    ve = np.ascontiguousarray(sc.var_edges, np.int32)
    nf = llr.shape[0]
    it = sc.n_iter if n_iter is None else n_iter
    d = LdpcC(N=sc.N, M=sc.M, dv=sc.dv, dc=sc.dc, n_frames=nf, n_iter=it,
              alpha=sc.alpha if alpha is None else alpha, nc_chk=sc.nc_chk, nc_var=sc.nc_var, check_vars=_ptr(cv),
              var_edges=_ptr(ve), llr=_ptr(llr))
    post = np.zeros((nf, sc.N), np.float32)
    err = np.zeros((nf, it), np.int32)
    if fn == "orc_ldpc_pipeline":
        st = Stats()
        assert lib().orc_ldpc_pipeline(C.byref(d), _ptr(post), _ptr(err), C.byref(st)) == 0
        return dict(post=post, errors=err, deq=list(st.deq[:4]), enq=list(st.enq[:4]))
    assert fn == "orc_ldpc_definition"
    assert lib().orc_ldpc_definition(C.byref(d), _ptr(post), _ptr(err)) == 0
    return dict(post=post, errors=err)


def ldpc_definition(sc, **kw):
    """LDPC min-sum decoder, definition layer (ldpc.c): posterior LLRs after the last
    iteration and bit errors per (frame, iteration)."""
    return _ldpc_run("orc_ldpc_definition", sc, **kw)


def ldpc_pipeline(sc, **kw):
    return _ldpc_run("orc_ldpc_pipeline", sc, **kw)


def collatz_definition(seeds: np.ndarray):
    seeds = np.ascontiguousarray(seeds)
    out = np.zeros(seeds.size, np.uint32)
    assert lib().orc_collatz_definition(_ptr(seeds), seeds.size, _ptr(out)) == 0
    return out


def collatz_pipeline(seeds: np.ndarray, max_steps: int = 1000):
    seeds = np.ascontiguousarray(seeds)
    out = np.zeros(seeds.size, np.uint32)
    seen = np.zeros(seeds.size, np.uint32)
    st = Stats()
    rc = lib().orc_collatz_pipeline(_ptr(seeds), seeds.size, max_steps, _ptr(out), _ptr(seen), C.byref(st))
    return rc, out, seen, list(st.deq[:2]), list(st.enq[:2])


# ------------------------------------------------------------------ Reyes
class _SceneHolder:
    """Keeps the numpy arrays referenced by the C struct alive."""

    def __init__(self, scene):
        self.M = np.ascontiguousarray(scene.M, np.float32).reshape(-1)
        self.albedo = np.ascontiguousarray(scene.albedo, np.float32).reshape(-1)
        s = ReyesSceneC()
        s.W, s.H, s.n_frames = scene.W, scene.H, scene.n_frames
        s.patches_per_frame = scene.patches_per_frame
        s.max_depth = scene.max_depth
        s.t_dice, s.near_w = scene.t_dice, scene.near_w
        s.M, s.albedo = self.M.ctypes.data, self.albedo.ctypes.data
        for i in range(4):
            s.L[i] = float(np.float32(scene.light[i]))
        self.c = s


def _reyes_run(fn, scene, seeds=None, leaf_cap=0, want_grids=False, trace_cap=0):
    seeds = np.ascontiguousarray(scene.seeds if seeds is None else seeds)
    h = _SceneHolder(scene)
    npix = scene.n_frames * scene.W * scene.H
    key = np.empty(npix, np.uint64)
    s = np.empty(npix, np.float32)
    colour = np.empty((npix, 4), np.float32)
    o = ReyesOutC()
    o.key, o.s, o.colour = key.ctypes.data, s.ctypes.data, colour.ctypes.data
    leaf_ids = np.zeros(max(leaf_cap, 1), np.uint64)
    grids = np.zeros((max(leaf_cap, 1) if want_grids else 1, 6, 81), np.float32)
    if leaf_cap:
        o.leaf_ids, o.leaf_cap = leaf_ids.ctypes.data, leaf_cap
        if want_grids:
            o.leaf_grids = grids.ctypes.data
    trace = np.zeros(max(trace_cap, 1), TRACE_DTYPE)
    if trace_cap:
        o.trace, o.trace_cap = trace.ctypes.data, trace_cap
    rc = fn(C.byref(h.c), _ptr(seeds), seeds.size, C.byref(o))
    assert rc == 0, rc
    shp = (scene.n_frames, scene.H, scene.W)
    res = dict(key=key.reshape(shp), s=s.reshape(shp), colour=colour.reshape(shp + (4,)),
               n_bound=o.n_bound, n_split=o.n_split, n_dice=o.n_dice, n_shade=o.n_shade,
               n_culled=o.n_culled, depth_hist=list(o.depth_hist),
               culled_depth_hist=list(o.culled_depth_hist), n_leaves=o.n_leaves, n_mp_covering=o.n_mp_covering)
    if leaf_cap:
        assert o.n_leaves <= leaf_cap, "leaf_cap too small"
        res["leaf_ids"] = leaf_ids[: o.n_leaves].copy()
        if want_grids:
            res["leaf_grids"] = grids[: o.n_leaves].copy()
    if trace_cap:
        assert o.trace_n <= trace_cap, "trace_cap too small"
        res["trace"] = trace[: o.trace_n].copy()
    return res


def reyes_definition(scene, seeds=None, leaf_cap=0, want_grids=False):
    return _reyes_run(lib().orc_reyes_definition, scene, seeds, leaf_cap, want_grids)


def reyes_pipeline(scene, seeds=None, leaf_cap=0, trace_cap=0):
    return _reyes_run(lib().orc_reyes_pipeline, scene, seeds, leaf_cap, False, trace_cap)


def reyes_bound(scene, patch_item):
    h = _SceneHolder(scene)
    it = np.ascontiguousarray(patch_item).reshape(1)
    d = C.c_int(0)
    cls = lib().orc_reyes_bound(C.byref(h.c), _ptr(it), C.byref(d))
    return cls, d.value


def reyes_split(patch_item, direction: int):
    it = np.ascontiguousarray(patch_item).reshape(1)
    left = np.zeros(1, it.dtype)
    right = np.zeros(1, it.dtype)
    lib().orc_reyes_split(_ptr(it), direction, _ptr(left), _ptr(right))
    return left[0], right[0]


def reyes_dice(scene, patch_item):
    h = _SceneHolder(scene)
    it = np.ascontiguousarray(patch_item).reshape(1)
    g = np.zeros((6, 81), np.float32)
    lib().orc_reyes_dice(C.byref(h.c), _ptr(it), _ptr(g))
    return g


def reyes_project(M16: np.ndarray, p4: np.ndarray):
    M = np.ascontiguousarray(M16, np.float32).reshape(16)
    p = np.ascontiguousarray(p4, np.float32).reshape(4)
    c = np.zeros(4, np.float32)
    lib().orc_reyes_project(_ptr(M), _ptr(p), _ptr(c))
    return c


def reyes_shade_factor(n3, L4):
    n = np.ascontiguousarray(n3, np.float32).reshape(3)
    L = np.ascontiguousarray(L4, np.float32).reshape(4)
    return float(lib().orc_reyes_shade_factor(_ptr(n), _ptr(L)))


REYES_CULL, REYES_SPLIT, REYES_DICE = 0, 1, 2


# ------------------------------------------------------------------ Rasterization
class RasterSceneC(C.Structure):
    _fields_ = [("W", C.c_int32), ("H", C.c_int32), ("n_tris", C.c_int64), ("M", P), ("pos", P), ("col", P),
                ("near_clip", C.c_int32)]


class RasterOutC(C.Structure):
    _fields_ = [("key", P), ("colour", P), ("n_vertex", C.c_uint64), ("n_clip", C.c_uint64),
                ("n_raster", C.c_uint64), ("n_fragment", C.c_uint64), ("n_frag_pixels", C.c_uint64),
                ("trace", P), ("trace_cap", C.c_size_t), ("trace_n", C.c_size_t)]


def _raster_run(fname, scene, trace_cap=0):
    L = lib()
    fn = getattr(L, fname)
    fn.argtypes = [P, P]
    M = np.ascontiguousarray(scene.M, np.float32).reshape(-1)
    pos = np.ascontiguousarray(scene.pos, np.float32)
    col = np.ascontiguousarray(scene.col, np.float32)
    sc = RasterSceneC(W=scene.W, H=scene.H, n_tris=pos.shape[0], M=M.ctypes.data, pos=pos.ctypes.data,
                      col=col.ctypes.data, near_clip=int(getattr(scene, "near_clip", 0)))
    npix = scene.W * scene.H
    key = np.empty(npix, np.uint64)
    colour = np.empty((npix, 4), np.float32)
    o = RasterOutC(key=key.ctypes.data, colour=colour.ctypes.data)
    trace = np.zeros(max(trace_cap, 1), TRACE_DTYPE)
    if trace_cap:
        o.trace, o.trace_cap = trace.ctypes.data, trace_cap
    rc = fn(C.byref(sc), C.byref(o))
    assert rc == 0, rc
    res = dict(key=key.reshape(scene.H, scene.W), colour=colour.reshape(scene.H, scene.W, 4),
               n_vertex=o.n_vertex, n_clip=o.n_clip, n_raster=o.n_raster, n_fragment=o.n_fragment,
               n_frag_pixels=o.n_frag_pixels)
    if trace_cap:
        assert o.trace_n <= trace_cap, "trace_cap too small"
        res["trace"] = trace[: o.trace_n].copy()
    return res


class PyrSceneC(C.Structure):
    _fields_ = [("S", C.c_int32), ("n_img", C.c_int32), ("rgb", P)]


class PyrOutC(C.Structure):
    _fields_ = [("gray", P), ("hist", P), ("lut", P), ("pyr", P), ("n_gray", C.c_uint64), ("n_cdf", C.c_uint64),
                ("n_map", C.c_uint64), ("n_resize", C.c_uint64), ("trace", P), ("trace_cap", C.c_size_t),
                ("trace_n", C.c_size_t)]


def pyr_levels(S):
    return lib().orc_pyr_levels(S)


def pyr_level_offset(S, l):
    f = lib().orc_pyr_level_offset
    f.restype = C.c_size_t
    return int(f(S, l))


def histeq_lut(hist, N):
    h = np.ascontiguousarray(hist, np.uint32)
    lut = np.zeros(256, np.uint8)
    f = lib().orc_histeq_lut
    f.argtypes = [P, C.c_uint64, P]
    f(_ptr(h), N, _ptr(lut))
    return lut


def _pyr_run(fname, rgb, trace_cap=0):
    rgb = np.ascontiguousarray(rgb, np.uint8)
    n, S = rgb.shape[0], rgb.shape[1]
    L = pyr_levels(S)
    total = pyr_level_offset(S, L)
    gray = np.zeros((n, S * S), np.uint8)
    hist = np.zeros((n, 256), np.uint32)
    lut = np.zeros((n, 256), np.uint8)
    pyr = np.zeros((n, total), np.uint8)
    sc = PyrSceneC(S=S, n_img=n, rgb=rgb.ctypes.data)
    o = PyrOutC(gray=gray.ctypes.data, hist=hist.ctypes.data, lut=lut.ctypes.data, pyr=pyr.ctypes.data)
    trace = np.zeros(max(trace_cap, 1), TRACE_DTYPE)
    if trace_cap:
        o.trace, o.trace_cap = trace.ctypes.data, trace_cap
    fn = getattr(lib(), fname)
    fn.argtypes = [P, P]
    rc = fn(C.byref(sc), C.byref(o))
    assert rc == 0, rc
    res = dict(gray=gray, hist=hist, lut=lut, pyr=pyr, n_gray=o.n_gray, n_cdf=o.n_cdf, n_map=o.n_map,
               n_resize=o.n_resize, levels=L)
    if trace_cap:
        res["trace"] = trace[: o.trace_n].copy()
    return res


def pyr_definition(rgb):
    return _pyr_run("orc_pyr_definition", rgb)


def pyr_pipeline(rgb, trace_cap=0):
    return _pyr_run("orc_pyr_pipeline", rgb, trace_cap)


class CfdSceneC(C.Structure):
    _fields_ = [("G", C.c_int32), ("T", C.c_int32), ("n_outer", C.c_int32), ("pad", C.c_int32), ("vars0", P),
                ("area", P), ("nb", P), ("normals", P), ("ff", C.c_float * 5)]


class CfdOutC(C.Structure):
    _fields_ = [("vars", P), ("n_copy", C.c_uint64), ("n_step", C.c_uint64), ("n_flux", C.c_uint64),
                ("n_time", C.c_uint64), ("trace", P), ("trace_cap", C.c_size_t), ("trace_n", C.c_size_t)]


def _cfd_run(fname, scene, n_outer=None, trace_cap=0):
    arrs = [np.ascontiguousarray(scene.vars0, np.float32), np.ascontiguousarray(scene.area, np.float32),
            np.ascontiguousarray(scene.nb, np.int32), np.ascontiguousarray(scene.normals, np.float32)]
    sc = CfdSceneC(G=scene.G, T=scene.T, n_outer=scene.n_outer if n_outer is None else n_outer,
                   vars0=arrs[0].ctypes.data, area=arrs[1].ctypes.data, nb=arrs[2].ctypes.data,
                   normals=arrs[3].ctypes.data)
    for i in range(5):
        sc.ff[i] = float(scene.ff[i])
    out = np.zeros((5, scene.G * scene.G), np.float32)
    o = CfdOutC(vars=out.ctypes.data)
    trace = np.zeros(max(trace_cap, 1), TRACE_DTYPE)
    if trace_cap:
        o.trace, o.trace_cap = trace.ctypes.data, trace_cap
    fn = getattr(lib(), fname)
    fn.argtypes = [P, P]
    rc = fn(C.byref(sc), C.byref(o))
    assert rc == 0, rc
    res = dict(vars=out, n_copy=o.n_copy, n_step=o.n_step, n_flux=o.n_flux, n_time=o.n_time)
    if trace_cap:
        res["trace"] = trace[: o.trace_n].copy()
    return res


def cfd_definition(scene, n_outer=None):
    return _cfd_run("orc_cfd_definition", scene, n_outer)


def cfd_pipeline(scene, n_outer=None, trace_cap=0):
    return _cfd_run("orc_cfd_pipeline", scene, n_outer, trace_cap)


class FdSceneC(C.Structure):
    _fields_ = [("W", C.c_int32), ("H", C.c_int32), ("n_frames", C.c_int32), ("n_stages", C.c_int32), ("rgb", P),
                ("n_weak", C.c_int32 * 16), ("thr", C.c_int32 * 16), ("weak", P)]


class FdOutC(C.Structure):
    _fields_ = [("levels", P), ("lbp", P), ("hist", P), ("lut", P), ("det", P), ("det_cap", C.c_size_t),
                ("n_det", C.c_size_t), ("survivors", C.c_uint64 * 16), ("windows", C.c_uint64),
                ("deq", C.c_uint64 * 8), ("trace", P), ("trace_cap", C.c_size_t), ("trace_n", C.c_size_t)]


def fd_levels(W, H):
    Ws, Hs = (C.c_int * 8)(), (C.c_int * 8)()
    L = lib().orc_fd_levels(W, H, Ws, Hs)
    return [(Ws[i], Hs[i]) for i in range(L)]


def _fd_run(fname, scene, det_cap=1 << 16, trace_cap=0):
    rgb = np.ascontiguousarray(scene.rgb, np.uint8)
    weak = np.ascontiguousarray(scene.weak, np.int32)
    sc = FdSceneC(W=scene.W, H=scene.H, n_frames=rgb.shape[0], n_stages=len(scene.n_weak), rgb=rgb.ctypes.data,
                  weak=weak.ctypes.data)
    for k, (n, t) in enumerate(zip(scene.n_weak, scene.thr)):
        sc.n_weak[k], sc.thr[k] = int(n), int(t)
    per = sum(w * h for w, h in fd_levels(scene.W, scene.H))
    F = rgb.shape[0]
    levels = np.zeros((F, per), np.uint8)
    lbp = np.zeros((F, per), np.uint8)
    hist = np.zeros((F, 256), np.uint32)
    lut = np.zeros((F, 256), np.uint8)
    det = np.zeros((det_cap, 4), np.uint32)
    o = FdOutC(levels=levels.ctypes.data, lbp=lbp.ctypes.data, hist=hist.ctypes.data, lut=lut.ctypes.data,
               det=det.ctypes.data, det_cap=det_cap)
    trace = np.zeros(max(trace_cap, 1), TRACE_DTYPE)
    if trace_cap:
        o.trace, o.trace_cap = trace.ctypes.data, trace_cap
    fn = getattr(lib(), fname)
    fn.argtypes = [P, P]
    rc = fn(C.byref(sc), C.byref(o))
    assert rc == 0, rc
    assert o.n_det <= det_cap
    res = dict(levels=levels, lbp=lbp, hist=hist, lut=lut, det=det[: o.n_det].copy(), n_det=o.n_det,
               survivors=list(o.survivors[: len(scene.n_weak)]), windows=o.windows, deq=list(o.deq[:6]))
    if trace_cap:
        res["trace"] = trace[: o.trace_n].copy()
    return res


def fd_definition(scene, det_cap=1 << 16):
    return _fd_run("orc_fd_definition", scene, det_cap)


def fd_pipeline(scene, det_cap=1 << 16, trace_cap=0):
    return _fd_run("orc_fd_pipeline", scene, det_cap, trace_cap)


def raster_definition(scene):
    return _raster_run("orc_raster_definition", scene)


def raster_pipeline(scene, trace_cap=0):
    return _raster_run("orc_raster_pipeline", scene, trace_cap)

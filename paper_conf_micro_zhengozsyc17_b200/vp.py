"""Thin ctypes binding of libvp.so (include/vp.h): argument marshalling only.

Every step of the pipeline runs in the CUDA kernels behind the C ABI.  There is no CPU
fallback: importing this module raises if libvp.so is missing or cannot be loaded.
PyTorch is used by callers only for device memory and streams; raw device pointers and
``cudaStream_t`` handles are what cross the ABI.
"""
from __future__ import annotations

import ctypes as C
import os

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.path.join(_HERE, os.environ.get("VP_LIB_NAME", "libvp.so"))

if not os.path.exists(LIB_PATH):
    raise ImportError(f"libvp.so not built at {LIB_PATH}: run `python -c 'import __graft_entry__ as g; g.build()'` "
                      "(there is no CPU fallback)")
_lib = C.CDLL(LIB_PATH)

MAX_STAGES = 8
MAX_SM = 256

# ---- enums (vp.h)
VP_OK, VP_ERR_INVALID, VP_ERR_UNSUPPORTED, VP_ERR_CUDA, VP_ERR_OOM, VP_ERR_QUEUE_OVERFLOW, VP_ERR_TIMEOUT, \
    VP_ERR_BINDING, VP_ERR_FANOUT = range(9)
RTC, KBK, MEGAKERNEL, COARSE, FINE, HYBRID, KBK_GRAPH = range(7)
MODEL_NAMES = {RTC: "rtc", KBK: "kbk", MEGAKERNEL: "megakernel", COARSE: "coarse", FINE: "fine", HYBRID: "hybrid",
               KBK_GRAPH: "kbk_graph"}
GROUP_RTC, GROUP_KBK, GROUP_MEGA, GROUP_FINE = range(4)
TOY_S1, TOY_S2, TOY_S3 = 1, 2, 3
COLLATZ_STEP, COLLATZ_SINK = 10, 11
REYES_BOUND, REYES_SPLIT, REYES_DICE, REYES_SHADE = 20, 21, 22, 23
RASTER_VERTEX, RASTER_CLIP, RASTER_RASTER, RASTER_FRAGMENT = 30, 31, 32, 33
PYR_GRAY, PYR_CDF, PYR_MAP, PYR_RESIZE = 40, 41, 42, 43
CFD_COPY, CFD_STEP_FACTOR, CFD_FLUX, CFD_TIME_STEP = 50, 51, 52, 53
FD_GRAY, FD_CDF, FD_MAP, FD_RESIZE, FD_LBP, FD_SCAN = 60, 61, 62, 63, 64, 65
QB_ITEM4, QB_ITEM16, QB_ITEM272 = 70, 71, 72
QB_ITEM4_CS, QB_ITEM16_CS = 73, 74
LDPC_INIT, LDPC_C2V, LDPC_V2C, LDPC_PROBVAR = 80, 81, 82, 83
FLAG_TRACE, FLAG_QUEUE_DEPTH, FLAG_STRICT_BINDING, FLAG_TIMERS, FLAG_FULL_RINGS, FLAG_ONLINE, FLAG_L2_PERSIST = (
    1, 2, 4, 8, 16, 32, 64)
FLAG_SERIALIZE_GROUPS, FLAG_NO_RERUN, FLAG_CLUSTER_STEAL = 0x80, 0x100, 0x200
INSERT_DEVICE, INSERT_REPLACE = 1, 2

P = C.c_void_p


class PipelineDesc(C.Structure):
    _fields_ = [("max_stages", C.c_int), ("flags", C.c_uint32), ("default_queue_capacity", C.c_int64),
                ("watchdog_ms", C.c_int), ("trace_capacity", C.c_int64)]


class StageDesc(C.Structure):
    _fields_ = [("name", C.c_char_p), ("kind", C.c_int), ("item_bytes", C.c_int), ("threads_per_item", C.c_int),
                ("queue_capacity", C.c_int64), ("params", P), ("params_bytes", C.c_size_t)]


class SmBinding(C.Structure):
    _fields_ = [("num_groups", C.c_int), ("group_of_stage", C.c_int * MAX_STAGES),
                ("group_model", C.c_int * MAX_STAGES),
                ("group_sm_mask", (C.c_uint32 * (MAX_SM // 32)) * MAX_STAGES),
                ("blocks_per_sm", C.c_int * MAX_STAGES), ("batch", C.c_int * MAX_STAGES)]


class Config(C.Structure):
    _fields_ = [("model", C.c_int), ("has_binding", C.c_int), ("binding", SmBinding), ("batch", C.c_int)]


class RunStats(C.Structure):
    _fields_ = [("device_ms", C.c_double), ("dequeued", C.c_uint64 * MAX_STAGES),
                ("enqueued", C.c_uint64 * MAX_STAGES), ("max_depth", C.c_uint64 * MAX_STAGES),
                ("num_kernels", C.c_int), ("kernel_lo", C.c_int * 16), ("kernel_hi", C.c_int * 16),
                ("kernel_quota", C.c_int * 16), ("kernel_ms", C.c_double * 16), ("blocks_on_sm", (C.c_uint32 * MAX_SM) * 16),
                ("admitted", C.c_uint64 * 16), ("fallback_admits", C.c_uint64), ("kbk_launches", C.c_uint64),
                ("trace_records", C.c_uint64), ("abort_reason", C.c_int), ("num_sms", C.c_int),
                ("stage_exec_ns", C.c_uint64 * MAX_STAGES), ("stage_flush_ns", C.c_uint64 * MAX_STAGES),
                ("kernel_idle_ns", C.c_uint64 * 16), ("ring_tail", C.c_uint64 * MAX_STAGES),
                ("ring_head", C.c_uint64 * MAX_STAGES), ("ring_count", C.c_int64 * MAX_STAGES),
                ("seed_head", C.c_uint64 * MAX_STAGES), ("pending", C.c_int64), ("kernel_rounds", C.c_uint64 * 16),
                ("stage_wave_ms", C.c_float * MAX_STAGES), ("dispatch_timeouts", C.c_int), ("model_rerun", C.c_int),
                ("work_units", C.c_uint64 * MAX_STAGES), ("stolen", C.c_uint64 * MAX_STAGES)]


class AutotuneOpts(C.Structure):
    _fields_ = [("time_budget_s", C.c_double), ("sm_granularity", C.c_int), ("batch_choices", C.c_int * 4),
                ("models_allowed", C.c_uint32), ("max_candidates", C.c_int), ("repeats", C.c_int)]


class TuneReport(C.Structure):
    _fields_ = [("candidates_total", C.c_int), ("candidates_run", C.c_int), ("candidates_timed_out", C.c_int),
                ("best_ms", C.c_double), ("baseline_kbk_ms", C.c_double), ("baseline_mega_ms", C.c_double),
                ("max_blocks_per_sm", C.c_int * MAX_STAGES), ("regs_per_thread", C.c_int * MAX_STAGES),
                ("smem_per_block", C.c_int * MAX_STAGES)]


class ToyParams(C.Structure):
    _fields_ = [("threshold", C.c_int32), ("pad", C.c_int32), ("out", P), ("n_out", P)]


class LdpcParams(C.Structure):
    _fields_ = [("N", C.c_int32), ("M", C.c_int32), ("dv", C.c_int32), ("dc", C.c_int32), ("n_frames", C.c_int32),
                ("n_iter", C.c_int32), ("alpha", C.c_float), ("nc_chk", C.c_int32), ("nc_var", C.c_int32),
                ("pad", C.c_int32), ("check_vars", P), ("var_edges", P), ("llr", P), ("v2c", P), ("c2v", P), ("post", P),
                ("errors", P), ("latch", P)]


class QBenchParams(C.Structure):
    _fields_ = [("fanout", C.c_uint32), ("depth", C.c_uint32), ("leaves", P), ("idsum", P), ("bad", P)]


class CollatzParams(C.Structure):
    _fields_ = [("steps_out", P), ("seen", P), ("n_ids", C.c_uint32), ("max_steps", C.c_uint32)]


class ReyesParams(C.Structure):
    _fields_ = [("W", C.c_int32), ("H", C.c_int32), ("n_frames", C.c_int32), ("patches_per_frame", C.c_int32),
                ("max_depth", C.c_int32), ("frame_base", C.c_int32), ("t_dice", C.c_float), ("near_w", C.c_float),
                ("M", P), ("albedo", P), ("L", C.c_float * 4), ("fb", P), ("colour", P)]


class RasterParams(C.Structure):
    _fields_ = [("W", C.c_int32), ("H", C.c_int32), ("n_tris", C.c_int64), ("M", P), ("pos", P), ("col", P),
                ("setup", P), ("fb", P), ("colour", P), ("near_clip", C.c_int32), ("pad0", C.c_int32),
                ("ccol", P)]


class PyramidParams(C.Structure):
    _fields_ = [("S", C.c_int32), ("n_img", C.c_int32), ("rgb", P), ("gray", P), ("pyr", P), ("hist", P),
                ("lut", P), ("latch", P)]


class CfdParams(C.Structure):
    _fields_ = [("G", C.c_int32), ("T", C.c_int32), ("n_outer", C.c_int32), ("pad0", C.c_int32), ("vars0", P),
                ("vars", P), ("old", P), ("sf", P), ("flux", P), ("area", P), ("nb", P), ("normals", P),
                ("ff", C.c_float * 5), ("pad1", C.c_int32), ("latch", P)]


class FaceDetParams(C.Structure):
    _fields_ = [("W", C.c_int32), ("H", C.c_int32), ("n_frames", C.c_int32), ("n_stages", C.c_int32),
                ("n_weak", C.c_int32 * 16), ("thr", C.c_int32 * 16), ("n_weak_total", C.c_int32),
                ("pad0", C.c_int32), ("rgb", P), ("levels", P), ("lbp", P), ("hist", P), ("lut", P), ("weak", P),
                ("det", P), ("det_count", P), ("det_cap", C.c_uint64), ("survivors", P), ("windows", P),
                ("latch", P)]


def _decl(name, args, res=C.c_int):
    f = getattr(_lib, name)
    f.argtypes = args
    f.restype = res
    return f


vp_status_string = _decl("vp_status_string", [C.c_int], C.c_char_p)
vp_last_error = _decl("vp_last_error", [P], C.c_char_p)
vp_pipeline_create = _decl("vp_pipeline_create", [C.c_int, C.POINTER(PipelineDesc), C.POINTER(P)])
vp_pipeline_destroy = _decl("vp_pipeline_destroy", [P])
vp_stage_register = _decl("vp_stage_register", [P, C.POINTER(StageDesc), C.POINTER(C.c_int)])
vp_insert = _decl("vp_insert", [P, C.c_int, P, C.c_size_t, C.c_int])
vp_insert_async = _decl("vp_insert_async", [P, C.c_int, P, C.c_size_t, C.c_int, P])
vp_configure = _decl("vp_configure", [P, C.c_int, C.POINTER(SmBinding), C.c_int])
vp_configure_config = _decl("vp_configure_config", [P, C.POINTER(Config)])
vp_get_config = _decl("vp_get_config", [P, C.POINTER(Config)])
vp_run = _decl("vp_run", [P, P, C.POINTER(RunStats)])
vp_set_timeout = _decl("vp_set_timeout", [P, C.c_double])
vp_get_trace = _decl("vp_get_trace", [P, C.POINTER(P), C.POINTER(C.c_size_t)])
vp_autotune = _decl("vp_autotune", [P, C.POINTER(AutotuneOpts), C.POINTER(Config), C.POINTER(TuneReport)])
vp_profile = _decl("vp_profile", [P, C.POINTER(C.c_int), C.POINTER(C.c_int), C.POINTER(C.c_int)])
vp_get_output = _decl("vp_get_output", [P, C.c_int, C.POINTER(P), C.POINTER(C.c_size_t)])
vp_set_params = _decl("vp_set_params", [P, P, C.c_size_t])
vp_config_to_string = _decl("vp_config_to_string", [C.POINTER(Config), C.c_char_p, C.c_size_t])
vp_config_from_string = _decl("vp_config_from_string", [C.c_char_p, C.POINTER(Config)])
vp_stage_kind_info = _decl("vp_stage_kind_info", [C.c_int, C.POINTER(C.c_int), C.POINTER(C.c_int)])
vp_device_info = _decl("vp_device_info", [C.c_int, C.POINTER(C.c_int), C.POINTER(C.c_int), C.POINTER(C.c_int)])
vp_memcpy = _decl("vp_memcpy", [P, P, C.c_size_t, C.c_int, P])
vp_set_flags = _decl("vp_set_flags", [P, C.c_uint32, C.POINTER(C.c_uint32)])
vp_bench_red_min_u64 = _decl("vp_bench_red_min_u64", [C.c_int, C.c_ulonglong, C.c_ulonglong, C.POINTER(C.c_double)])

EXPORTED = ["vp_status_string", "vp_last_error", "vp_pipeline_create", "vp_pipeline_destroy", "vp_stage_register",
            "vp_insert", "vp_insert_async", "vp_configure", "vp_configure_config", "vp_get_config", "vp_run",
            "vp_set_timeout", "vp_get_trace", "vp_autotune", "vp_profile", "vp_get_output", "vp_set_params", "vp_config_to_string", "vp_config_from_string",
            "vp_device_info", "vp_memcpy", "vp_set_flags", "vp_bench_red_min_u64", "vp_stage_kind_info"]


class VPError(RuntimeError):
    def __init__(self, status, msg):
        super().__init__(f"{vp_status_string(status).decode()}: {msg}")
        self.status = status


def _ptr_of(x):
    """device/host address of a torch tensor or numpy array (no copies)."""
    if hasattr(x, "data_ptr"):
        return C.c_void_p(x.data_ptr())
    if isinstance(x, np.ndarray):
        assert x.flags["C_CONTIGUOUS"]
        return C.c_void_p(x.ctypes.data)
    if isinstance(x, int):
        return C.c_void_p(x)
    raise TypeError(type(x))


def _stream_handle(stream):
    if stream is None:
        return None
    if hasattr(stream, "cuda_stream"):
        return C.c_void_p(stream.cuda_stream)
    return C.c_void_p(int(stream))


def stage_kind_info(kind):
    """vp_stage_kind_info: (item_bytes, threads_per_item) a built-in stage kind is registered with."""
    b, t = C.c_int(), C.c_int()
    rc = vp_stage_kind_info(kind, C.byref(b), C.byref(t))
    if rc != VP_OK:
        raise VPError(rc, f"vp_stage_kind_info({kind})")
    return b.value, t.value


def device_info(device=0):
    n, a, b = C.c_int(), C.c_int(), C.c_int()
    rc = vp_device_info(device, C.byref(n), C.byref(a), C.byref(b))
    if rc != VP_OK:
        raise VPError(rc, "vp_device_info")
    return n.value, (a.value, b.value)


def bench_red_min_u64(slots, n_ops=1 << 30, device=0):
    """vp_bench_red_min_u64: measured 64-bit atomic-min (RED) rate into a `slots`-entry buffer."""
    r = C.c_double(0.0)
    rc = vp_bench_red_min_u64(device, slots, n_ops, C.byref(r))
    if rc != VP_OK:
        raise VPError(rc, "vp_bench_red_min_u64")
    return r.value


def make_binding(groups, num_sms, blocks_per_sm=None, batch=None):
    """groups: list of (stage_lo, stage_hi, group_model, sm_lo, sm_hi) -> SmBinding."""
    b = SmBinding()
    b.num_groups = len(groups)
    for g, (lo, hi, model, sm_lo, sm_hi) in enumerate(groups):
        for s in range(lo, hi + 1):
            b.group_of_stage[s] = g
        b.group_model[g] = model
        for sm in range(sm_lo, min(sm_hi, num_sms)):
            b.group_sm_mask[g][sm >> 5] |= 1 << (sm & 31)
    for s, v in enumerate(blocks_per_sm or []):
        b.blocks_per_sm[s] = v
    for s, v in enumerate(batch or []):
        b.batch[s] = v
    return b


class Pipeline:
    def __init__(self, device=0, flags=0, queue_capacity=0, watchdog_ms=0, trace_capacity=0):
        d = PipelineDesc(max_stages=MAX_STAGES, flags=flags, default_queue_capacity=queue_capacity,
                         watchdog_ms=watchdog_ms, trace_capacity=trace_capacity)
        h = P()
        rc = vp_pipeline_create(device, C.byref(d), C.byref(h))
        if rc != VP_OK:
            raise VPError(rc, f"vp_pipeline_create(device={device})")
        self.h = h
        self.device = device
        self.trace_capacity = trace_capacity if trace_capacity > 0 else (1 << 20)
        self._keep = []

    def _check(self, rc, what):
        if rc != VP_OK:
            raise VPError(rc, f"{what}: {vp_last_error(self.h).decode()}")

    def register(self, kind, item_bytes, params=None, threads_per_item=0, queue_capacity=0, name=None):
        sd = StageDesc(name=(name or f"kind{kind}").encode(), kind=kind, item_bytes=item_bytes,
                       threads_per_item=threads_per_item, queue_capacity=queue_capacity,
                       params=C.cast(C.byref(params), P) if params is not None else None,
                       params_bytes=C.sizeof(params) if params is not None else 0)
        sid = C.c_int(-1)
        self._check(vp_stage_register(self.h, C.byref(sd), C.byref(sid)), "vp_stage_register")
        return sid.value

    def insert(self, stage, items, n=None, replace=False, stream=None):
        on_dev = hasattr(items, "is_cuda") and items.is_cuda
        if n is None:
            n = items.shape[0] if hasattr(items, "shape") else len(items)
        flags = (INSERT_DEVICE if on_dev else 0) | (INSERT_REPLACE if replace else 0)
        if stream is None:
            self._check(vp_insert(self.h, stage, _ptr_of(items), n, flags), "vp_insert")
        else:
            self._check(vp_insert_async(self.h, stage, _ptr_of(items), n, flags, _stream_handle(stream)),
                        "vp_insert_async")

    def configure(self, model, binding=None, batch=0):
        self._check(vp_configure(self.h, model, C.byref(binding) if binding is not None else None, batch),
                    "vp_configure")

    def configure_config(self, cfg):
        self._check(vp_configure_config(self.h, C.byref(cfg)), "vp_configure_config")

    def get_config(self):
        c = Config()
        self._check(vp_get_config(self.h, C.byref(c)), "vp_get_config")
        return c

    def run(self, stream=None, raw=False):
        st = RunStats()
        self._check(vp_run(self.h, _stream_handle(stream), C.byref(st)), "vp_run")
        return st if raw else stats_dict(st)

    def run_status(self, stream=None):
        st = RunStats()
        rc = vp_run(self.h, _stream_handle(stream), C.byref(st))
        return rc, stats_dict(st), vp_last_error(self.h).decode()

    def trace_ptr(self):
        ptr, n = P(), C.c_size_t()
        self._check(vp_get_trace(self.h, C.byref(ptr), C.byref(n)), "vp_get_trace")
        return ptr.value

    TRACE_DTYPE = np.dtype([("id", "<u8"), ("stage", "<u4"), ("smid", "<u4"), ("kslot", "<u4"), ("block", "<u4")])

    def trace(self, stats):
        """The last run's task trace (VP_FLAG_TRACE) copied to the host: one record per
        task {id, stage, smid, kslot, block} (vp.h vp_get_trace)."""
        n = min(int(stats["trace_records"]), int(self.trace_capacity))
        host = np.zeros(n, self.TRACE_DTYPE)
        if n:
            rc = vp_memcpy(C.c_void_p(host.ctypes.data), C.c_void_p(self.trace_ptr()), host.nbytes, 1, None)
            self._check(rc, "vp_memcpy(trace)")
        return host

    def set_flags(self, flags):
        """Run-time flags (FLAG_QUEUE_DEPTH | FLAG_STRICT_BINDING | FLAG_TIMERS | FLAG_SERIALIZE_GROUPS |
        FLAG_NO_RERUN);
        returns the previous flags."""
        old = C.c_uint32()
        self._check(vp_set_flags(self.h, flags, C.byref(old)), "vp_set_flags")
        return old.value

    def set_timeout_ms(self, ms):
        self._check(vp_set_timeout(self.h, float(ms)), "vp_set_timeout")

    def profile(self, n_stages):
        mb = (C.c_int * MAX_STAGES)()
        rg = (C.c_int * MAX_STAGES)()
        sm = (C.c_int * MAX_STAGES)()
        self._check(vp_profile(self.h, mb, rg, sm), "vp_profile")
        return list(mb[:n_stages]), list(rg[:n_stages]), list(sm[:n_stages])

    def autotune(self, time_budget_s=30.0, sm_granularity=0, batch_choices=(1,), models_allowed=0,
                 max_candidates=0, repeats=1):
        o = AutotuneOpts(time_budget_s=time_budget_s, sm_granularity=sm_granularity, models_allowed=models_allowed,
                         max_candidates=max_candidates, repeats=repeats)
        for i, b in enumerate(list(batch_choices)[:4]):
            o.batch_choices[i] = b
        best = Config()
        rep = TuneReport()
        self._check(vp_autotune(self.h, C.byref(o), C.byref(best), C.byref(rep)), "vp_autotune")
        return best, rep

    def set_params(self, params):
        """vp_set_params: replace the family parameter struct between runs."""
        self._check(vp_set_params(self.h, C.cast(C.byref(params), P), C.sizeof(params)), "vp_set_params")

    def output(self, index):
        ptr, n = P(), C.c_size_t()
        self._check(vp_get_output(self.h, index, C.byref(ptr), C.byref(n)), "vp_get_output")
        return ptr.value, n.value

    def close(self):
        if getattr(self, "h", None):
            vp_pipeline_destroy(self.h)
            self.h = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass


def stats_dict(st: RunStats):
    nk = st.num_kernels
    return dict(device_ms=st.device_ms, dequeued=list(st.dequeued), enqueued=list(st.enqueued),
                max_depth=list(st.max_depth), num_kernels=nk,
                kernels=[(st.kernel_lo[i], st.kernel_hi[i], st.kernel_quota[i]) for i in range(nk)],
                kernel_ms=list(st.kernel_ms[:nk]),
                blocks_on_sm=[list(st.blocks_on_sm[i][:st.num_sms]) for i in range(max(nk, 1))],
                admitted=list(st.admitted[:nk]), fallback_admits=st.fallback_admits,
                kbk_launches=st.kbk_launches, trace_records=st.trace_records, abort_reason=st.abort_reason,
                num_sms=st.num_sms, stage_exec_ns=list(st.stage_exec_ns), stage_flush_ns=list(st.stage_flush_ns),
                kernel_idle_ns=list(st.kernel_idle_ns[:max(nk, 1)]), ring_tail=list(st.ring_tail),
                ring_head=list(st.ring_head), ring_count=list(st.ring_count), seed_head=list(st.seed_head),
                pending=st.pending, kernel_rounds=list(st.kernel_rounds[:max(nk, 1)]),
                stage_wave_ms=list(st.stage_wave_ms), dispatch_timeouts=st.dispatch_timeouts,
                model_rerun=st.model_rerun, work_units=list(st.work_units), stolen=list(st.stolen))


def config_to_string(cfg: Config) -> str:
    buf = C.create_string_buffer(8192)
    rc = vp_config_to_string(C.byref(cfg), buf, len(buf))
    if rc != VP_OK:
        raise VPError(rc, "vp_config_to_string")
    return buf.value.decode()


def config_from_string(s: str) -> Config:
    c = Config()
    rc = vp_config_from_string(s.encode(), C.byref(c))
    if rc != VP_OK:
        raise VPError(rc, "vp_config_from_string")
    return c

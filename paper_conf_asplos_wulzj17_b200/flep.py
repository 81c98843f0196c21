"""Thin ctypes binding of include/flep.h — argument marshalling only.

Every step of the hot path runs in libflep.so (the CUDA kernels and the C++ runtime). PyTorch is
used by callers only for device memory and streams. There is no CPU fallback: importing this
module on a machine without the built library raises.
"""
from __future__ import annotations

import ctypes as C
import os

HERE = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.environ.get("FLEP_LIB_PATH") or os.path.join(HERE, "libflep.so")   # override: A/B builds

OK, ERR_INVALID, ERR_STATE, ERR_CUDA, ERR_NOMEM, ERR_TIMEOUT, ERR_UNSUPPORTED = 0, -1, -2, -3, -4, -5, -6
POLICY_MANUAL, POLICY_FIFO, POLICY_HPF, POLICY_SLICE, POLICY_FFS, POLICY_REORDER = 0, 1, 2, 3, 4, 5
POLICY_SLICE_DEVICE = 6
FLAG_STREAM_MEMOP, FLAG_HOST_MAPPED = 0, 1
BODY_SAXPY_I32, BODY_SAXPY_F32, BODY_SPMV_CSR_F32, BODY_STENCIL5_F32, BODY_STENCIL5_I32, BODY_GEMM_BF16 = 1, 2, 3, 4, 5, 6
BODY_STENCIL5_F32_TMA = 7
BODY_SPMV_CSR_F32_VEC = 8
BODY_GEMM_BF16_2SM = 9
BODY_GEMM_BF16_2SM_W = 10
STATE_QUEUED, STATE_RUNNING, STATE_YIELDING, STATE_PREEMPTED, STATE_PARTIAL, STATE_DONE = 0, 1, 2, 3, 4, 5
STATE_NAMES = {0: "QUEUED", 1: "RUNNING", 2: "YIELDING", 3: "PREEMPTED", 4: "PARTIAL", 5: "DONE"}
REASON_YIELD, REASON_EXHAUSTED = 1, 2
RELAY_LEFT_OWN_SM, RELAY_LEFT_TEMPORAL, RELAY_LEFT_PUBLISHED = 1, 2, 3
ACTION_NAMES = {0: "LAUNCH", 1: "RESUME", 2: "PREEMPT", 3: "REFILL"}
NO_TRIGGER = 0xFFFFFFFF
KFLAG_PREFETCH = 1
KFLAG_STARTED_HINT = 2
KFLAG_IN_TILE = 4
KFLAG_ASYNC_POLL = 8
KFLAG_CLC = 16
KFLAG_SCHED_WARP = 32
KFLAG_HOST_RELAY = 64
KFLAG_WARP_TASKS = 128
KFLAG_IN_CHUNK = 256
KFLAG_SPEC_FETCH = 512
WARP_TASKS_PER_BLOCK = 8


class Dim3(C.Structure):
    _fields_ = [("x", C.c_uint32), ("y", C.c_uint32), ("z", C.c_uint32)]


class SaxpyI32Args(C.Structure):
    _fields_ = [("y", C.c_void_p), ("x", C.c_void_p), ("a", C.c_int32), ("n", C.c_uint32)]


class SaxpyF32Args(C.Structure):
    _fields_ = [("y", C.c_void_p), ("x", C.c_void_p), ("a", C.c_float), ("n", C.c_uint32)]


class SpmvArgs(C.Structure):
    _fields_ = [("y", C.c_void_p), ("rowptr", C.c_void_p), ("col", C.c_void_p), ("val", C.c_void_p),
                ("x", C.c_void_p), ("rows", C.c_uint32)]


class StencilArgs(C.Structure):
    _fields_ = [("out", C.c_void_p), ("inp", C.c_void_p), ("n", C.c_uint32)]


class GemmArgs(C.Structure):
    _fields_ = [("c", C.c_void_p), ("a", C.c_void_p), ("b", C.c_void_p), ("m", C.c_uint32),
                ("n", C.c_uint32), ("k", C.c_uint32)]


class Options(C.Structure):
    _fields_ = [("policy", C.c_int32), ("flag", C.c_int32), ("default_chunk", C.c_uint32),
                ("default_poll", C.c_uint32), ("debug_coverage", C.c_uint32),
                ("spatial", C.c_uint32), ("slice_blocks", C.c_uint32),
                ("exec_on_user_stream", C.c_uint32), ("max_overhead_ppm", C.c_uint32)]


class KernelDesc(C.Structure):
    _fields_ = [("name", C.c_char_p), ("body", C.c_int32), ("chunk", C.c_uint32), ("poll", C.c_uint32),
                ("model", C.c_double * 5), ("preempt_overhead_ns", C.c_int64), ("flags", C.c_uint32),
                ("ctas_per_sm", C.c_uint32)]


class LaunchInfo(C.Structure):
    _fields_ = [("state", C.c_int32), ("epoch", C.c_uint32), ("blocks_total", C.c_uint64),
                ("blocks_done", C.c_uint64), ("counter", C.c_uint64), ("t_e", C.c_int64),
                ("t_w", C.c_int64), ("t_r", C.c_int64), ("t_arrive", C.c_int64),
                ("t_first_start", C.c_int64), ("t_finish", C.c_int64), ("workers", C.c_uint32),
                ("n_yield", C.c_uint32), ("t_last_request", C.c_int64), ("t_last_drain", C.c_int64),
                ("started_epoch", C.c_uint32), ("tasks_per_block", C.c_uint32)]


class WorkerEvent(C.Structure):
    _fields_ = [("smid", C.c_uint32), ("reason", C.c_uint32), ("n_blocks", C.c_uint32),
                ("epoch", C.c_uint32), ("t_entry", C.c_uint64), ("t_exit", C.c_uint64)]


class BodyOps(C.Structure):
    """flep_body_ops (include/flep.h): filled by a user body library's `<sym>_ops` function."""
    _fields_ = [("abi_version", C.c_uint32), ("threads", C.c_uint32), ("args_size", C.c_size_t),
                ("name", C.c_char_p), ("worker", C.c_void_p), ("unwrapped", C.c_void_p),
                ("static_launch", C.c_void_p), ("occupancy", C.c_void_p), ("clc", C.c_void_p),
                ("sliced", C.c_void_p)]


BODY_USER_FIRST = 64


class EpochInfo(C.Structure):
    _fields_ = [("t_trigger", C.c_uint64), ("t_end", C.c_uint64), ("trigger_block", C.c_uint32),
                ("done", C.c_uint32), ("counter", C.c_uint32), ("state", C.c_uint32),
                ("relay_smid", C.c_uint32), ("relay_reason", C.c_uint32), ("relay_t_exit", C.c_uint64)]


ARGS_FOR_BODY = {BODY_SAXPY_I32: SaxpyI32Args, BODY_SAXPY_F32: SaxpyF32Args, BODY_SPMV_CSR_F32: SpmvArgs,
                 BODY_STENCIL5_F32: StencilArgs, BODY_STENCIL5_I32: StencilArgs, BODY_GEMM_BF16: GemmArgs,
                 BODY_STENCIL5_F32_TMA: StencilArgs, BODY_SPMV_CSR_F32_VEC: SpmvArgs, BODY_GEMM_BF16_2SM: GemmArgs,
                 BODY_GEMM_BF16_2SM_W: GemmArgs}

# exported symbols: name -> (restype, argtypes)
_P = C.c_void_p
_SIG = {
    "flep_init": (C.c_int, [C.c_int, C.POINTER(Options), C.POINTER(_P)]),
    "flep_shutdown": (C.c_int, [_P]),
    "flep_device_info": (C.c_int, [_P, C.POINTER(C.c_uint32), C.POINTER(C.c_uint32)]),
    "flep_register_kernel": (C.c_int, [_P, C.POINTER(KernelDesc), C.POINTER(C.c_int32)]),
    "flep_register_body": (C.c_int, [_P, C.POINTER(BodyOps), C.POINTER(C.c_int32)]),
    "flep_launch": (C.c_int, [_P, C.c_int32, Dim3, _P, C.c_size_t, C.c_int32, _P, C.POINTER(C.c_int64)]),
    "flep_preempt": (C.c_int, [_P, C.c_int64, C.c_uint32]),
    "flep_resume": (C.c_int, [_P, C.c_int64]),
    "flep_refill": (C.c_int, [_P, C.c_int64]),
    "flep_sync": (C.c_int, [_P, C.c_int64, C.c_int64]),
    "flep_query": (C.c_int, [_P, C.c_int64, C.POINTER(LaunchInfo)]),
    "flep_cancel": (C.c_int, [_P, C.c_int64]),
    "flep_wait_epoch": (C.c_int, [_P, C.c_int64, C.c_int64]),
    "flep_launch_unwrapped": (C.c_int, [_P, C.c_int32, Dim3, _P, C.c_size_t, _P]),
    "flep_launch_sliced": (C.c_int, [_P, C.c_int32, Dim3, _P, C.c_size_t, C.c_uint32, _P]),
    "flep_launch_static": (C.c_int, [_P, C.c_int32, Dim3, _P, C.c_size_t, C.c_uint32, _P]),
    "flep_workers_for": (C.c_int, [_P, C.c_int32, C.POINTER(C.c_uint32), C.POINTER(C.c_uint32)]),
    "flep_debug_trigger_at": (C.c_int, [_P, C.c_int64, C.c_uint64, C.c_uint32]),
    "flep_debug_arm_next_trigger": (C.c_int, [_P, C.c_uint64, C.c_uint32]),
    "flep_debug_copy_coverage": (C.c_int, [_P, C.c_int64, C.POINTER(C.c_uint32), C.c_size_t]),
    "flep_debug_copy_events": (C.c_int, [_P, C.c_int64, C.c_uint32, C.POINTER(WorkerEvent), C.c_size_t,
                                         C.POINTER(C.c_size_t)]),
    "flep_debug_epoch_info": (C.c_int, [_P, C.c_int64, C.c_uint32, C.POINTER(EpochInfo)]),
    "flep_debug_set_trace": (C.c_int, [_P, C.c_void_p, C.c_void_p]),
    "flep_set_rank_table": (C.c_int, [_P, C.POINTER(C.c_uint16), C.c_uint32]),
    "flep_now_ns": (C.c_int64, []),
    "flep_decision_log": (C.c_int, [_P, C.POINTER(C.c_int64), C.c_size_t, C.POINTER(C.c_size_t)]),
    "flep_event_log": (C.c_int, [_P, C.POINTER(C.c_int64), C.c_size_t, C.POINTER(C.c_size_t)]),
    "flep_event_log_ex": (C.c_int, [_P, C.POINTER(C.c_int64), C.c_size_t, C.POINTER(C.c_size_t)]),
    "flep_policy_create": (C.c_int, [C.c_int32, C.c_uint32, C.POINTER(_P)]),
    "flep_policy_destroy": (C.c_int, [_P]),
    "flep_policy_arrive": (C.c_int, [_P, C.c_int64, C.c_int64, C.c_int32, C.c_int64, C.c_int64]),
    "flep_policy_arrive_ex": (C.c_int, [_P, C.c_int64, C.c_int64, C.c_int32, C.c_int64, C.c_int64, C.c_int64]),
    "flep_policy_set_spatial": (C.c_int, [_P, C.c_int32]),
    "flep_policy_finish": (C.c_int, [_P, C.c_int64, C.c_int64]),
    "flep_policy_decisions": (C.c_int, [_P, C.POINTER(C.c_int64), C.c_size_t, C.POINTER(C.c_size_t)]),
    "flep_policy_tick": (C.c_int, [_P, C.c_int64, C.POINTER(C.c_int32)]),
    "flep_policy_set_max_overhead": (C.c_int, [_P, C.c_uint32]),
    "flep_model_predict_ns": (C.c_int64, [C.POINTER(C.c_double), C.c_double, C.c_double, C.c_double,
                                          C.c_double]),
    "flep_last_error": (C.c_char_p, []),
    "flep_version": (C.c_char_p, []),
}

_lib = None


_user_libs = {}                       # user body libraries, loaded once and never unloaded


def lib():
    """Load libflep.so (raises if it is missing — there is no fallback)."""
    global _lib
    if _lib is None:
        if not os.path.exists(LIB_PATH):
            raise RuntimeError(f"{LIB_PATH} is missing: run `python -m paper_conf_asplos_wulzj17_b200.build` "
                               "(the FLEP path has no CPU fallback)")
        L = C.CDLL(LIB_PATH)
        for name, (res, args) in _SIG.items():
            f = getattr(L, name)
            f.restype = res
            f.argtypes = args
        _lib = L
    return _lib


class FlepError(RuntimeError):
    def __init__(self, status, where):
        msg = lib().flep_last_error().decode(errors="replace")
        super().__init__(f"{where}: status {status}: {msg}")
        self.status = status


def check(status, where=""):
    if status != OK:
        raise FlepError(status, where)
    return status


def _stream_ptr(stream):
    if stream is None:
        return None
    if isinstance(stream, int):
        return stream
    return stream.cuda_stream  # torch.cuda.Stream


def dim3(g):
    if isinstance(g, int):
        return Dim3(g, 1, 1)
    g = tuple(g) + (1,) * (3 - len(g))
    return Dim3(*g)


class Runtime:
    """One FLEP runtime on one device (flep_init ... flep_shutdown)."""

    def __init__(self, device=0, policy=POLICY_MANUAL, flag=FLAG_STREAM_MEMOP, chunk=8, poll=1,
                 coverage=False, slice_blocks=0, exec_on_user_stream=False, max_overhead_ppm=0, spatial=False,
                 keep_logs=False):
        self.L = lib()
        dbg = 1 if coverage else (2 if keep_logs else 0)
        o = Options(policy, flag, chunk, poll, dbg, int(spatial), slice_blocks,
                    int(exec_on_user_stream), max_overhead_ppm)
        h = C.c_void_p()
        check(self.L.flep_init(device, C.byref(o), C.byref(h)), "flep_init")
        self.h = h
        n, ns = C.c_uint32(), C.c_uint32()
        check(self.L.flep_device_info(self.h, C.byref(n), C.byref(ns)), "flep_device_info")
        self.num_sms, self.nsmid = n.value, ns.value

    def close(self):
        if self.h:
            check(self.L.flep_shutdown(self.h), "flep_shutdown")
            self.h = None

    def __enter__(self):
        return self

    def __exit__(self, *a):
        self.close()

    def register_kernel(self, body, chunk=0, poll=0, name="", model=(0, 0, 0, 0, 1), overhead_ns=0,
                        prefetch=False, ctas_per_sm=0, started_hint=False, in_tile=False, async_poll=False,
                        clc=False, sched_warp=False, host_relay=False, warp_tasks=False, in_chunk=False,
                        spec_fetch=False):
        flags = ((KFLAG_PREFETCH if prefetch else 0) | (KFLAG_STARTED_HINT if started_hint else 0)
                 | (KFLAG_IN_TILE if in_tile else 0) | (KFLAG_ASYNC_POLL if async_poll else 0)
                 | (KFLAG_CLC if clc else 0) | (KFLAG_SCHED_WARP if sched_warp else 0)
                 | (KFLAG_HOST_RELAY if host_relay else 0) | (KFLAG_WARP_TASKS if warp_tasks else 0)
                 | (KFLAG_IN_CHUNK if in_chunk else 0) | (KFLAG_SPEC_FETCH if spec_fetch else 0))
        d = KernelDesc(name.encode(), body, chunk, poll, (C.c_double * 5)(*model), overhead_ns,
                       flags, ctas_per_sm)
        k = C.c_int32()
        check(self.L.flep_register_kernel(self.h, C.byref(d), C.byref(k)), "flep_register_kernel")
        return k.value

    def register_body(self, lib_path, sym):
        """Register a user-defined body (include/flep_body.cuh): load its library (kept loaded
        for the process), fill the ops table through `<sym>_ops` and return the body id."""
        ul = _user_libs.get(lib_path)
        if ul is None:
            ul = _user_libs[lib_path] = C.CDLL(lib_path)
        fill = getattr(ul, sym + "_ops")
        fill.restype = None
        fill.argtypes = [C.POINTER(BodyOps)]
        ops = BodyOps()
        fill(C.byref(ops))
        body = C.c_int32()
        check(self.L.flep_register_body(self.h, C.byref(ops), C.byref(body)), "flep_register_body")
        return body.value

    def launch(self, kernel, grid, args, priority=0, stream=None):
        out = C.c_int64()
        check(self.L.flep_launch(self.h, kernel, dim3(grid), C.byref(args), C.sizeof(args), priority,
                                 _stream_ptr(stream), C.byref(out)), "flep_launch")
        return out.value

    def preempt(self, launch, n_sms):
        check(self.L.flep_preempt(self.h, launch, n_sms), "flep_preempt")

    def resume(self, launch):
        check(self.L.flep_resume(self.h, launch), "flep_resume")

    def refill(self, launch):
        check(self.L.flep_refill(self.h, launch), "flep_refill")

    def sync(self, launch, timeout_ns=-1):
        check(self.L.flep_sync(self.h, launch, timeout_ns), "flep_sync")

    def wait_epoch(self, launch, timeout_ns=-1):
        check(self.L.flep_wait_epoch(self.h, launch, timeout_ns), "flep_wait_epoch")

    def cancel(self, launch):
        check(self.L.flep_cancel(self.h, launch), "flep_cancel")

    def query(self, launch):
        i = LaunchInfo()
        check(self.L.flep_query(self.h, launch, C.byref(i)), "flep_query")
        return i

    def launch_unwrapped(self, body, grid, args, stream=None):
        check(self.L.flep_launch_unwrapped(self.h, body, dim3(grid), C.byref(args), C.sizeof(args),
                                           _stream_ptr(stream)), "flep_launch_unwrapped")

    def launch_sliced(self, body, grid, args, slice_blocks, stream=None):
        check(self.L.flep_launch_sliced(self.h, body, dim3(grid), C.byref(args), C.sizeof(args),
                                        slice_blocks, _stream_ptr(stream)), "flep_launch_sliced")

    def launch_static(self, body, grid, args, chunk=1, stream=None):
        check(self.L.flep_launch_static(self.h, body, dim3(grid), C.byref(args), C.sizeof(args), chunk,
                                        _stream_ptr(stream)), "flep_launch_static")

    def workers_for(self, body):
        k, w = C.c_uint32(), C.c_uint32()
        check(self.L.flep_workers_for(self.h, body, C.byref(k), C.byref(w)), "flep_workers_for")
        return k.value, w.value

    def trigger_at(self, launch, block, n_sms):
        check(self.L.flep_debug_trigger_at(self.h, launch, block, n_sms), "flep_debug_trigger_at")

    def arm_next_trigger(self, block, n_sms):
        check(self.L.flep_debug_arm_next_trigger(self.h, block, n_sms), "flep_debug_arm_next_trigger")

    def coverage(self, launch, n):
        buf = (C.c_uint32 * n)()
        check(self.L.flep_debug_copy_coverage(self.h, launch, buf, n), "flep_debug_copy_coverage")
        return list(buf)

    def coverage_np(self, launch, n):
        import numpy as np
        a = np.zeros(n, dtype=np.uint32)
        check(self.L.flep_debug_copy_coverage(self.h, launch, a.ctypes.data_as(C.POINTER(C.c_uint32)), n),
              "flep_debug_copy_coverage")
        return a

    def events(self, launch, epoch):
        info = self.query(launch)
        buf = (WorkerEvent * max(1, info.workers))()
        n = C.c_size_t()
        check(self.L.flep_debug_copy_events(self.h, launch, epoch, buf, info.workers, C.byref(n)),
              "flep_debug_copy_events")
        return [buf[i] for i in range(n.value)]

    def epoch_info(self, launch, epoch):
        e = EpochInfo()
        check(self.L.flep_debug_epoch_info(self.h, launch, epoch, C.byref(e)), "flep_debug_epoch_info")
        return e

    def set_trace(self, worker_trace=None, unwrapped_trace=None):
        """Diagnostics builds (-DFLEP_TRACE) only: device buffers (torch tensors) for the chunk /
        block timestamp traces, or None."""
        ptr = lambda t: None if t is None else C.c_void_p(t.data_ptr())  # noqa: E731
        check(self.L.flep_debug_set_trace(self.h, ptr(worker_trace), ptr(unwrapped_trace)), "flep_debug_set_trace")

    def set_rank_table(self, rank):
        arr = (C.c_uint16 * len(rank))(*rank)
        check(self.L.flep_set_rank_table(self.h, arr, len(rank)), "flep_set_rank_table")

    def decision_log(self):
        n = C.c_size_t()
        check(self.L.flep_decision_log(self.h, None, 0, C.byref(n)), "flep_decision_log")
        buf = (C.c_int64 * (4 * max(1, n.value)))()
        check(self.L.flep_decision_log(self.h, buf, n.value, C.byref(n)), "flep_decision_log")
        return [tuple(buf[4 * i:4 * i + 4]) for i in range(n.value)]

    def event_log(self):
        n = C.c_size_t()
        check(self.L.flep_event_log(self.h, None, 0, C.byref(n)), "flep_event_log")
        buf = (C.c_int64 * (6 * max(1, n.value)))()
        check(self.L.flep_event_log(self.h, buf, n.value, C.byref(n)), "flep_event_log")
        return [tuple(buf[6 * i:6 * i + 6]) for i in range(n.value)]

    def event_log_ex(self):
        """(t, type, launch, priority, t_e, overhead, sms_need) records."""
        n = C.c_size_t()
        check(self.L.flep_event_log_ex(self.h, None, 0, C.byref(n)), "flep_event_log_ex")
        buf = (C.c_int64 * (7 * max(1, n.value)))()
        check(self.L.flep_event_log_ex(self.h, buf, n.value, C.byref(n)), "flep_event_log_ex")
        return [tuple(buf[7 * i:7 * i + 7]) for i in range(n.value)]


def now_ns():
    return lib().flep_now_ns()


class PolicyEngine:
    """The runtime's pure decision engine (flep_policy_*), host only."""

    def __init__(self, kind, num_sms=148, spatial=False):
        self.L = lib()
        h = C.c_void_p()
        check(self.L.flep_policy_create(kind, num_sms, C.byref(h)), "flep_policy_create")
        self.h = h
        if spatial:
            check(self.L.flep_policy_set_spatial(self.h, 1), "flep_policy_set_spatial")

    def __del__(self):
        if getattr(self, "h", None):
            self.L.flep_policy_destroy(self.h)
            self.h = None

    def arrive(self, t, kid, prio, t_e, overhead, sms_need=0):
        check(self.L.flep_policy_arrive_ex(self.h, t, kid, prio, t_e, overhead, sms_need), "flep_policy_arrive_ex")

    def finish(self, t, kid):
        check(self.L.flep_policy_finish(self.h, t, kid), "flep_policy_finish")

    def tick(self, t):
        a = C.c_int32()
        check(self.L.flep_policy_tick(self.h, t, C.byref(a)), "flep_policy_tick")
        return bool(a.value)

    def set_max_overhead(self, ppm):
        check(self.L.flep_policy_set_max_overhead(self.h, ppm), "flep_policy_set_max_overhead")

    def decisions(self):
        n = C.c_size_t()
        check(self.L.flep_policy_decisions(self.h, None, 0, C.byref(n)), "flep_policy_decisions")
        buf = (C.c_int64 * (4 * max(1, n.value)))()
        check(self.L.flep_policy_decisions(self.h, buf, n.value, C.byref(n)), "flep_policy_decisions")
        return [tuple(buf[4 * i:4 * i + 4]) for i in range(n.value)]


def model_predict_ns(model5, grid, cta, inp, smem):
    m = (C.c_double * 5)(*model5)
    return lib().flep_model_predict_ns(m, grid, cta, inp, smem)


# ---- argument builders from torch tensors (pointers only; no compute) ------------------------
def saxpy_i32_args(y, x, a):
    return SaxpyI32Args(y.data_ptr(), x.data_ptr(), int(a), y.numel())


def saxpy_f32_args(y, x, a):
    return SaxpyF32Args(y.data_ptr(), x.data_ptr(), float(a), y.numel())


def spmv_args(y, rowptr, col, val, x):
    return SpmvArgs(y.data_ptr(), rowptr.data_ptr(), col.data_ptr(), val.data_ptr(), x.data_ptr(), y.numel())


def stencil_args(out, inp):
    return StencilArgs(out.data_ptr(), inp.data_ptr(), inp.shape[0])


def gemm_args(c, a, b):
    return GemmArgs(c.data_ptr(), a.data_ptr(), b.data_ptr(), a.shape[0], b.shape[0], a.shape[1])


def saxpy_grid(n):
    return ((n + 255) // 256, 1, 1)


SPMV_ROWS_PER_BLOCK = int(os.environ.get("FLEP_SPMV_ROWS", "128"))   # = FLEP_SPMV_ROWS of the build


def spmv_grid(rows):
    return ((rows + SPMV_ROWS_PER_BLOCK - 1) // SPMV_ROWS_PER_BLOCK, 1, 1)


def stencil_grid(n):
    t = (n + 63) // 64
    return (t, t, 1)


def gemm_grid(m, n):
    return (n // 256, m // 128, 1)


def gemm2_grid(m, n):
    """Original grid of the CTA-pair GEMM body: one 256x256 tile per block."""
    return (n // 256, m // 256, 1)


def gemm2w_grid(m, n):
    """Original grid of the wide CTA-pair GEMM body: one 256x512 tile per block."""
    return (n // 512, m // 256, 1)

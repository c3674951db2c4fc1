"""Python binding of libpipedream.so (the B200-native PipeDream hot path).

Argument marshalling only: every step of the path (planner, schedule, kernels, transport)
runs inside the C-ABI library declared in ``include/pipedream.h``.  Function names mirror
the C names.  There is no fallback: if the shared library is missing, importing this
package raises, and without a B200 every device call raises ``PDError``.
"""
from __future__ import annotations

import ctypes as C
import os
from dataclasses import dataclass
from typing import List, Optional, Sequence

import numpy as np

# one hardware queue per worker stream; must be set
# before the CUDA context is created
os.environ.setdefault("CUDA_DEVICE_MAX_CONNECTIONS", "32")

_HERE = os.path.dirname(os.path.abspath(__file__))
# PD_LIBRARY: the negative-control tests point a subprocess at a fault-injected build
# (build.py FAULTS); the product path always loads the in-tree libpipedream.so
LIB_PATH = os.environ.get("PD_LIBRARY") or os.path.join(_HERE, "libpipedream.so")

PD_OK, PD_EINVAL, PD_ENOMEM, PD_ECUDA, PD_ENCCL, PD_ESTATE, PD_EUNSUPPORTED, PD_EINFEASIBLE = 0, -1, -2, -3, -4, -5, -6, -7
PD_LINEAR, PD_LSTM, PD_CONV3X3, PD_MAXPOOL2, PD_EMBEDDING = 0, 1, 2, 3, 4
PD_ACT_NONE, PD_ACT_RELU = 0, 1
PD_FP32, PD_BF16 = 0, 1
PD_SGD, PD_ADAM = 0, 1
PD_SYNC_STASH, PD_SYNC_VERTICAL, PD_SYNC_GPIPE = 0, 1, 2
PD_EPI_STORE, PD_EPI_MASK, PD_EPI_F32, PD_EPI_SGD, PD_EPI_ADAM = 0, 1, 2, 3, 4
PD_MAX_STAGES = 64
PD_MAX_LOCAL_WORKERS = 64
PD_KERNEL_CLASSES = 8
KERNEL_CLASSES = ["fwd_gemm", "dx_gemm", "dw_gemm", "other", "lstm_wave_fwd", "lstm_wave_bwd", "softmax_ce",
                  "optimizer_update"]


class PDError(RuntimeError):
    def __init__(self, status, msg=""):
        super().__init__(f"{status} ({_strerror(status)}){': ' + msg if msg else ''}")
        self.status = status


class LayerProfile(C.Structure):
    _fields_ = [("compute_s", C.c_double), ("act_bytes", C.c_uint64), ("param_bytes", C.c_uint64)]


PD_MAX_LEVELS = 4


class PlanOpts(C.Structure):
    _fields_ = [("bandwidth_Bps", C.c_double), ("max_replicas", C.c_int), ("comm_model", C.c_int),
                ("num_levels", C.c_int), ("level_size", C.c_int * PD_MAX_LEVELS),
                ("level_bw", C.c_double * PD_MAX_LEVELS)]


class StageDesc(C.Structure):
    _fields_ = [("first_layer", C.c_int), ("last_layer", C.c_int), ("replicas", C.c_int), ("first_gpu", C.c_int)]


class PlanT(C.Structure):
    _fields_ = [("num_stages", C.c_int), ("stage", StageDesc * PD_MAX_STAGES), ("noam", C.c_int),
                ("slowest_stage_s", C.c_double)]


class LayerDesc(C.Structure):
    _fields_ = [("kind", C.c_int), ("in_", C.c_int), ("out", C.c_int), ("act", C.c_int), ("seq_len", C.c_int),
                ("height", C.c_int), ("width", C.c_int)]


class TrainCfg(C.Structure):
    _fields_ = [("dtype", C.c_int), ("optimizer", C.c_int), ("lr", C.c_float), ("beta1", C.c_float),
                ("beta2", C.c_float), ("eps", C.c_float), ("minibatch", C.c_int), ("record_trace", C.c_int),
                ("max_depth", C.c_int), ("sync_mode", C.c_int)]


class Event(C.Structure):
    _fields_ = [("worker", C.c_int16), ("stage", C.c_int16), ("replica", C.c_int16), ("kind", C.c_int16),
                ("seq", C.c_int32), ("minibatch", C.c_int32), ("version_in", C.c_int32),
                ("version_out", C.c_int32), ("start_us", C.c_float), ("end_us", C.c_float)]


class Stats(C.Structure):
    _fields_ = [("host_ms", C.c_double), ("device_ms", C.c_double), ("bubble", C.c_double),
                ("kernel_launches", C.c_uint64), ("bytes_sent", C.c_uint64), ("num_local_workers", C.c_int),
                ("worker_id", C.c_int * PD_MAX_LOCAL_WORKERS), ("busy_ms", C.c_double * PD_MAX_LOCAL_WORKERS),
                ("span_ms", C.c_double * PD_MAX_LOCAL_WORKERS), ("run_ms", C.c_double),
                ("kern_ms", C.c_double * PD_KERNEL_CLASSES), ("kern_count", C.c_uint64 * PD_KERNEL_CLASSES),
                ("replica_bytes", C.c_uint64)]


class LstmRecDesc(C.Structure):
    _fields_ = [("direction", C.c_int), ("T", C.c_int), ("B", C.c_int), ("H", C.c_int), ("gx", C.c_void_p),
                ("b_ih", C.c_void_p), ("b_hh", C.c_void_p), ("w_hh", C.c_void_p), ("gates", C.c_void_p),
                ("c", C.c_void_p), ("h", C.c_void_p), ("dy", C.c_void_p), ("da", C.c_void_p),
                ("counters", C.c_void_p), ("probe", C.c_void_p)]


class GemmDesc(C.Structure):
    _fields_ = [("dtype", C.c_int), ("M", C.c_int), ("N", C.c_int), ("K", C.c_int), ("A", C.c_void_p),
                ("lda", C.c_long), ("a_mn_major", C.c_int), ("B", C.c_void_p), ("ldb", C.c_long),
                ("b_mn_major", C.c_int), ("epilogue", C.c_int), ("out", C.c_void_p), ("ldo", C.c_long),
                ("bias", C.c_void_p), ("relu", C.c_int), ("mask", C.c_void_p), ("ldm", C.c_long),
                ("master", C.c_void_p), ("slot", C.c_void_p), ("adam_m", C.c_void_p), ("adam_v", C.c_void_p),
                ("lr", C.c_float), ("beta1", C.c_float), ("beta2", C.c_float), ("eps", C.c_float),
                ("step", C.c_int), ("workspace", C.c_void_p), ("workspace_bytes", C.c_long),
                ("workspace_zeroed", C.c_int)]


def _load():
    if not os.path.exists(LIB_PATH):
        raise ImportError(f"{LIB_PATH} is missing: run __graft_entry__.build() (no CPU fallback exists)")
    L = C.CDLL(LIB_PATH)
    vp, i, st = C.c_void_p, C.c_int, C.c_size_t
    sigs = {
        "pd_plan": [vp, i, i, vp, vp],
        "pd_create": [vp, vp, vp, i, vp],
        "pd_stage_init": [vp, i, i, i, vp],
        "pd_export_worker": [vp, i, i, vp, st, vp],
        "pd_import_worker": [vp, vp, st],
        "pd_set_data": [vp, vp, vp, vp, i],
        "pd_run": [vp, i, i],
        "pd_get_params": [vp, i, vp, st],
        "pd_get_trace": [vp, vp, st, vp],
        "pd_get_version_map": [vp, vp, st],
        "pd_get_losses": [vp, vp, st],
        "pd_get_stats": [vp, vp],
        "pd_inflight": [vp, i, vp],
        "pd_set_timing": [vp, i, i],
        "pd_kernel_gemm": [vp, vp],
        "pd_kernel_softmax_ce": [i, vp, vp, C.c_long, i, vp, vp, vp],
        "pd_kernel_lstm_rec": [vp, vp],
        "pd_kernel_bias_grad": [i, vp, C.c_long, C.c_long, vp, vp, vp, i, vp, vp, C.c_float, C.c_float, C.c_float,
                                C.c_float, i, vp],
        "pd_profile": [vp, i, vp, i, i, vp],
        "pd_set_layer_profiling": [vp, i],
        "pd_get_layer_times": [vp, vp, vp, st],
        "pd_stage_solo": [vp],
        "pd_save_checkpoint": [vp, C.c_char_p],
        "pd_load_checkpoint": [vp, C.c_char_p],
    }
    for name, args in sigs.items():
        f = getattr(L, name)
        f.argtypes = args
        f.restype = C.c_int
    L.pd_destroy.argtypes = [vp]
    L.pd_destroy.restype = None
    L.pd_strerror.argtypes = [i]
    L.pd_strerror.restype = C.c_char_p
    L.pd_last_error.argtypes = [vp]
    L.pd_last_error.restype = C.c_char_p
    return L


lib = _load()

EXPORTED = ["pd_plan", "pd_create", "pd_stage_init", "pd_export_worker", "pd_import_worker", "pd_set_data", "pd_run",
            "pd_get_params", "pd_get_trace", "pd_get_version_map", "pd_get_losses", "pd_get_stats", "pd_destroy",
            "pd_strerror", "pd_last_error", "pd_inflight", "pd_kernel_gemm", "pd_kernel_softmax_ce",
            "pd_kernel_lstm_rec", "pd_profile", "pd_set_layer_profiling", "pd_get_layer_times",
            "pd_set_timing", "pd_kernel_bias_grad", "pd_stage_solo", "pd_save_checkpoint", "pd_load_checkpoint"]


def _strerror(s):
    return lib.pd_strerror(int(s)).decode()


def _check(s, ctx=None):
    if s != PD_OK:
        msg = lib.pd_last_error(ctx).decode() if ctx else ""
        raise PDError(s, msg)


def _ptr(a):
    return None if a is None else a.ctypes.data_as(C.c_void_p)


# ---------------------------------------------------------------------------------- planner

@dataclass
class Plan:
    stages: List[tuple]  # (first_layer, last_layer, replicas, first_gpu)
    noam: int
    slowest_stage_s: float

    @property
    def stage_last(self):
        return [s[1] for s in self.stages]

    @property
    def replicas(self):
        return [s[2] for s in self.stages]

    def to_c(self) -> PlanT:
        p = PlanT()
        p.num_stages = len(self.stages)
        for q, (a, b, r, g) in enumerate(self.stages):
            p.stage[q] = StageDesc(a, b, r, g)
        p.noam = self.noam
        p.slowest_stage_s = self.slowest_stage_s
        return p

    @staticmethod
    def from_c(p: PlanT) -> "Plan":
        st = [(p.stage[q].first_layer, p.stage[q].last_layer, p.stage[q].replicas, p.stage[q].first_gpu)
              for q in range(p.num_stages)]
        return Plan(st, p.noam, p.slowest_stage_s)

    @staticmethod
    def manual(stage_last: Sequence[int], replicas: Sequence[int]) -> "Plan":
        st, first, gpu = [], 0, 0
        for last, r in zip(stage_last, replicas):
            st.append((first, int(last), int(r), gpu))
            first, gpu = int(last) + 1, gpu + int(r)
        plan = Plan(st, 0, 0.0)
        plan.noam = pd_inflight(plan)[0]  # the library derives NOAM = k_0 (R1)
        return plan


def pd_plan(compute_s, act_bytes, param_bytes, num_gpus, bandwidth_Bps=0.0, max_replicas=0, comm_model=0,
            levels=None) -> Plan:
    """levels: optional [(m_1, B_1), ..., (m_L, B_L)] hierarchy (Fig. 7), lowest level first."""
    n = len(compute_s)
    prof = (LayerProfile * n)()
    for k in range(n):
        prof[k] = LayerProfile(float(compute_s[k]), int(act_bytes[k]), int(param_bytes[k]))
    opts = PlanOpts(bandwidth_Bps, max_replicas, comm_model)
    if levels:
        if len(levels) > PD_MAX_LEVELS:
            raise ValueError("too many topology levels")
        opts.num_levels = len(levels)
        for k, (m, bw) in enumerate(levels):
            opts.level_size[k] = int(m)
            opts.level_bw[k] = float(bw)
    out = PlanT()
    _check(lib.pd_plan(prof, n, num_gpus, C.byref(opts), C.byref(out)))
    return Plan.from_c(out)


def pd_profile(layers, dtype=PD_BF16, optimizer=PD_SGD, lr=0.01, minibatch=1, device=0, num_minibatches=8,
               beta1=0.9, beta2=0.999, eps=1e-8):
    """The B200 self-profiler (L841-847): (T_l seconds, a_l bytes, w_l bytes) per layer,
    measured on `device` by the library."""
    n = len(layers)
    out = (LayerProfile * n)()
    cfg = TrainCfg(dtype, optimizer, lr, beta1, beta2, eps, minibatch, 0, 0, 0)
    _check(lib.pd_profile(_layer_descs(layers), n, C.byref(cfg), device, num_minibatches, out))
    return ([out[k].compute_s for k in range(n)], [int(out[k].act_bytes) for k in range(n)],
            [int(out[k].param_bytes) for k in range(n)])


def pd_inflight(plan: Plan, noam: int = 0) -> List[int]:
    k = (C.c_int * len(plan.stages))()
    _check(lib.pd_inflight(C.byref(plan.to_c()), noam, k))
    return list(k)


# ---------------------------------------------------------------------------------- runtime

def _layer_descs(layers):
    arr = (LayerDesc * len(layers))()
    for k, L in enumerate(layers):
        t = L.as_tuple() if hasattr(L, "as_tuple") else tuple(L)
        arr[k] = LayerDesc(*t)
    return arr


def pd_create(plan: Plan, layers, dtype=PD_BF16, optimizer=PD_SGD, lr=0.01, beta1=0.9, beta2=0.999, eps=1e-8,
              minibatch=1, record_trace=1, max_depth=0, sync_mode=0):
    """sync_mode: PD_SYNC_STASH (weight stashing), PD_SYNC_VERTICAL (vertical sync, §3.3) or
    PD_SYNC_GPIPE (the §5.4 flush schedule with gradient aggregation, R27)."""
    ctx = C.c_void_p()
    cfg = TrainCfg(dtype, optimizer, lr, beta1, beta2, eps, minibatch, record_trace, max_depth, sync_mode)
    _check(lib.pd_create(C.byref(ctx), C.byref(plan.to_c()), _layer_descs(layers), len(layers), C.byref(cfg)))
    return ctx


def pd_stage_init(ctx, stage: int, replica: int, device: int, params: Sequence[Optional[np.ndarray]]):
    keep = [None if p is None or np.asarray(p).size == 0 else np.ascontiguousarray(p, np.float32) for p in params]
    arr = (C.c_void_p * max(1, len(keep)))()
    for k, p in enumerate(keep):
        arr[k] = None if p is None else p.ctypes.data
    _check(lib.pd_stage_init(ctx, stage, replica, device, arr), ctx)


def pd_export_worker(ctx, stage: int, replica: int) -> bytes:
    n = C.c_size_t(0)
    lib.pd_export_worker(ctx, stage, replica, None, 0, C.byref(n))
    buf = (C.c_char * n.value)()
    _check(lib.pd_export_worker(ctx, stage, replica, buf, n.value, C.byref(n)), ctx)
    return bytes(buf)


def pd_import_worker(ctx, blob: bytes):
    b = (C.c_char * len(blob)).from_buffer_copy(blob)
    _check(lib.pd_import_worker(ctx, b, len(blob)), ctx)


def _host_ptr(a, dtype):
    """numpy array -> (keepalive, pointer); a pinned torch CPU tensor is passed through."""
    if a is None:
        return None, None
    if hasattr(a, "data_ptr"):  # torch tensor (possibly pinned)
        return a, C.c_void_p(a.data_ptr())
    a = np.ascontiguousarray(a, dtype)
    return a, a.ctypes.data_as(C.c_void_p)


def pd_set_data(ctx, inputs, tokens, labels, num_minibatches: int):
    ki, pi = _host_ptr(inputs, np.float32)
    kt, pt = _host_ptr(tokens, np.int32)
    kl, pl = _host_ptr(labels, np.int32)
    _check(lib.pd_set_data(ctx, pi, pt, pl, num_minibatches), ctx)


def pd_run(ctx, num_minibatches: int, noam: int = 0):
    _check(lib.pd_run(ctx, num_minibatches, noam), ctx)


def pd_get_params(ctx, layer: int, count: int) -> np.ndarray:
    out = np.zeros(max(count, 1), np.float32)
    _check(lib.pd_get_params(ctx, layer, _ptr(out), count), ctx)
    return out[:count]


def pd_get_trace(ctx):
    n = C.c_size_t(0)
    _check(lib.pd_get_trace(ctx, None, 0, C.byref(n)), ctx)
    buf = (Event * max(1, n.value))()
    _check(lib.pd_get_trace(ctx, buf, n.value, C.byref(n)), ctx)
    return [(e.worker, e.stage, e.replica, e.seq, chr(e.kind), e.minibatch, e.version_in, e.version_out,
             e.start_us, e.end_us) for e in buf[:n.value]]


def pd_get_version_map(ctx, num_stages: int, M: int) -> np.ndarray:
    out = np.zeros(num_stages * M, np.int32)
    _check(lib.pd_get_version_map(ctx, _ptr(out), out.size), ctx)
    return out.reshape(num_stages, M)


def pd_get_losses(ctx, M: int) -> np.ndarray:
    out = np.zeros(M, np.float32)
    _check(lib.pd_get_losses(ctx, _ptr(out), M), ctx)
    return out


def pd_get_stats(ctx) -> dict:
    s = Stats()
    _check(lib.pd_get_stats(ctx, C.byref(s)), ctx)
    n = s.num_local_workers
    return {"host_ms": s.host_ms, "device_ms": s.device_ms, "bubble": s.bubble,
            "kernel_launches": int(s.kernel_launches), "bytes_sent": int(s.bytes_sent), "num_local_workers": n,
            "worker_id": list(s.worker_id[:n]), "busy_ms": list(s.busy_ms[:n]), "span_ms": list(s.span_ms[:n]),
            "run_ms": s.run_ms, "kern_ms": list(s.kern_ms), "kern_count": [int(x) for x in s.kern_count],
            "replica_bytes": int(s.replica_bytes)}


def pd_set_timing(ctx, record_trace: int, kernel_timing_mask: int = 0xFF):
    _check(lib.pd_set_timing(ctx, record_trace, kernel_timing_mask), ctx)


def pd_set_layer_profiling(ctx, on: bool):
    _check(lib.pd_set_layer_profiling(ctx, int(bool(on))), ctx)


def pd_get_layer_times(ctx, num_layers: int):
    """(forward seconds, backward seconds) per layer, mean per minibatch of the last run."""
    f = np.zeros(num_layers, np.float64)
    b = np.zeros(num_layers, np.float64)
    _check(lib.pd_get_layer_times(ctx, _ptr(f), _ptr(b), num_layers), ctx)
    return f, b


def pd_save_checkpoint(ctx, directory: str):
    """Every local worker writes <dir>/stage<s>_replica<r>.pdckpt (L1407-1413)."""
    _check(lib.pd_save_checkpoint(ctx, os.fsencode(directory)), ctx)


def pd_load_checkpoint(ctx, directory: str):
    _check(lib.pd_load_checkpoint(ctx, os.fsencode(directory)), ctx)


def pd_stage_solo(ctx):
    """Solo measurement mode: absent workers become stand-ins, local receive rings synthetic."""
    _check(lib.pd_stage_solo(ctx), ctx)


def pd_destroy(ctx):
    lib.pd_destroy(ctx)


def pd_strerror(status: int) -> str:
    return _strerror(status)


def pd_last_error(ctx) -> str:
    return lib.pd_last_error(ctx).decode()


# ---------------------------------------------------------------------------------- kernels

def pd_kernel_gemm(dtype, M, N, K, A, lda, B, ldb, out=None, ldo=0, a_mn_major=0, b_mn_major=0,
                   epilogue=PD_EPI_STORE, bias=None, relu=0, mask=None, ldm=0, master=None, slot=None,
                   adam_m=None, adam_v=None, lr=0.0, beta1=0.9, beta2=0.999, eps=1e-8, step=1, stream=None,
                   workspace=None, workspace_bytes=0, workspace_zeroed=0):
    """All array arguments are device addresses (ints), e.g. torch ``tensor.data_ptr()``."""
    d = GemmDesc(dtype, M, N, K, A, lda, a_mn_major, B, ldb, b_mn_major, epilogue, out, ldo, bias, relu, mask, ldm,
                 master, slot, adam_m, adam_v, lr, beta1, beta2, eps, step, workspace, workspace_bytes,
                 workspace_zeroed)
    _check(lib.pd_kernel_gemm(C.byref(d), stream))


def pd_kernel_bias_grad(dtype, G, rows, cols, grad_out=None, master=None, slot=None, optimizer=PD_SGD, m=None,
                        v=None, lr=0.0, beta1=0.9, beta2=0.999, eps=1e-8, step=1, stream=None):
    """db = column sums of G (device addresses as ints), written or applied as the update."""
    _check(lib.pd_kernel_bias_grad(dtype, G, rows, cols, grad_out, master, slot, optimizer, m, v, lr, beta1, beta2,
                                   eps, step, stream))


def pd_kernel_softmax_ce(dtype, logits, labels, rows, Cn, dlogits, loss, stream=None):
    _check(lib.pd_kernel_softmax_ce(dtype, logits, labels, rows, Cn, dlogits, loss, stream))


def pd_kernel_lstm_rec(direction, T, B, H, w_hh, gates, c, counters, gx=None, b_ih=None, b_hh=None, h=None,
                       dy=None, da=None, probe=None, stream=None):
    """One LSTM layer's recurrence in one persistent launch (device addresses as ints)."""
    d = LstmRecDesc(direction, T, B, H, gx, b_ih, b_hh, w_hh, gates, c, h, dy, da, counters, probe)
    _check(lib.pd_kernel_lstm_rec(C.byref(d), stream))

"""CPU oracle of PipeDream 1F1B + weight stashing -- TEST INFRASTRUCTURE ONLY.

Only ``tests/``, ``__graft_entry__.smoke()`` and ``bench.py``'s ``cpu_baseline`` /
``--impl reference`` legs may import this package.  The product path
(``paper_conf_sosp_narayananhpsdgg19_b200``) never imports it and shares no code with it.

This file is argument marshalling (ctypes) around ``oracle.cpp``; all arithmetic lives
there, written step by step from /root/reference/PAPER.md (see its header).
"""
from __future__ import annotations

import ctypes as C
import os
import subprocess
from dataclasses import dataclass
from typing import List, Optional, Sequence

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "oracle.cpp")
_LIB = os.path.join(_HERE, "liboracle.so")


class OrcLayer(C.Structure):
    _fields_ = [("kind", C.c_int), ("in_", C.c_int), ("out", C.c_int), ("act", C.c_int),
                ("seq_len", C.c_int), ("height", C.c_int), ("width", C.c_int)]


class OrcEvent(C.Structure):
    _fields_ = [("worker", C.c_int), ("stage", C.c_int), ("replica", C.c_int), ("seq", C.c_int),
                ("kind", C.c_int), ("minibatch", C.c_int), ("version_in", C.c_int),
                ("version_out", C.c_int), ("start", C.c_double), ("end", C.c_double)]


def build(force: bool = False) -> str:
    """Compile oracle.cpp (plain -O2, no -march, no fp contraction) into liboracle.so."""
    if force or not os.path.exists(_LIB) or os.path.getmtime(_LIB) < os.path.getmtime(_SRC):
        tmp = _LIB + f".tmp{os.getpid()}"
        subprocess.check_call(["g++", "-O2", "-std=c++17", "-ffp-contract=off", "-fPIC", "-shared",
                               "-o", tmp, _SRC])
        os.replace(tmp, _LIB)
    return _LIB


_lib = None


def lib():
    global _lib
    if _lib is None:
        build()
        L = C.CDLL(_LIB)
        L.orc_param_count.restype = C.c_long
        L.orc_in_size.restype = C.c_long
        L.orc_out_size.restype = C.c_long
        L.orc_softmax_ce.restype = C.c_float
        L.orc_softmax_ce.argtypes = [C.c_void_p, C.c_void_p, C.c_long, C.c_int, C.c_void_p]
        L.orc_update.argtypes = [C.c_int, C.c_float, C.c_float, C.c_float, C.c_float, C.c_void_p,
                                 C.c_void_p, C.c_void_p, C.c_void_p, C.c_long, C.c_int]
        L.orc_run.argtypes = [C.c_void_p, C.c_int, C.c_void_p, C.c_void_p, C.c_int, C.c_int, C.c_int,
                              C.c_int, C.c_int, C.c_float, C.c_float, C.c_float, C.c_float, C.c_int,
                              C.c_void_p, C.c_void_p, C.c_void_p, C.c_int, C.c_void_p, C.c_void_p,
                              C.c_void_p, C.c_void_p, C.c_int, C.c_void_p, C.c_void_p, C.c_void_p,
                              C.c_void_p, C.c_void_p, C.c_void_p]
        L.orc_plan.argtypes = [C.c_void_p, C.c_void_p, C.c_void_p, C.c_int, C.c_int, C.c_double,
                               C.c_int, C.c_int, C.c_void_p, C.c_void_p, C.c_void_p, C.c_void_p,
                               C.c_void_p]
        L.orc_plan_levels.argtypes = [C.c_void_p, C.c_void_p, C.c_void_p, C.c_int, C.c_int, C.c_void_p, C.c_void_p,
                                      C.c_int, C.c_int, C.c_void_p, C.c_void_p, C.c_void_p, C.c_void_p, C.c_void_p]
        _lib = L
    return _lib


def _ptr(a):
    return None if a is None else a.ctypes.data_as(C.c_void_p)


def _layers(layers) -> C.Array:
    arr = (OrcLayer * len(layers))()
    for i, L in enumerate(layers):
        arr[i] = OrcLayer(*L.as_tuple())
    return arr


def param_count(L) -> int:
    return int(lib().orc_param_count(C.byref(OrcLayer(*L.as_tuple()))))


def out_size(L, B) -> int:
    return int(lib().orc_out_size(C.byref(OrcLayer(*L.as_tuple())), B))


def in_size(L, B) -> int:
    return int(lib().orc_in_size(C.byref(OrcLayer(*L.as_tuple())), B))


def layer_forward(L, B, params, x=None, tokens=None):
    y = np.zeros(out_size(L, B), np.float32)
    params = np.ascontiguousarray(params, np.float32)
    x = None if x is None else np.ascontiguousarray(x, np.float32)
    tokens = None if tokens is None else np.ascontiguousarray(tokens, np.int32)
    lib().orc_layer_forward(C.byref(OrcLayer(*L.as_tuple())), B, _ptr(params), _ptr(x), _ptr(tokens), _ptr(y))
    return y


def layer_backward(L, B, params, x, tokens, dy, need_dx=True):
    params = np.ascontiguousarray(params, np.float32)
    x = None if x is None else np.ascontiguousarray(x, np.float32)
    tokens = None if tokens is None else np.ascontiguousarray(tokens, np.int32)
    dy = np.ascontiguousarray(dy, np.float32)
    dx = np.zeros(in_size(L, B), np.float32) if need_dx else None
    dp = np.zeros(max(1, len(params)), np.float32)
    lib().orc_layer_backward(C.byref(OrcLayer(*L.as_tuple())), B, _ptr(params), _ptr(x), _ptr(tokens),
                             _ptr(dy), _ptr(dx), _ptr(dp))
    return dx, dp[:len(params)]


def softmax_ce(logits, labels):
    logits = np.ascontiguousarray(logits, np.float32)
    labels = np.ascontiguousarray(labels, np.int32)
    R, Cn = logits.shape
    d = np.zeros_like(logits)
    loss = lib().orc_softmax_ce(_ptr(logits), _ptr(labels), R, Cn, _ptr(d))
    return float(loss), d


def update(kind, lr, w, g, m=None, v=None, step=1, b1=0.9, b2=0.999, eps=1e-8):
    w = np.array(w, np.float32)
    g = np.ascontiguousarray(g, np.float32)
    m = np.zeros_like(w) if m is None else np.array(m, np.float32)
    v = np.zeros_like(w) if v is None else np.array(v, np.float32)
    lib().orc_update(kind, lr, b1, b2, eps, _ptr(w), _ptr(g), _ptr(m), _ptr(v), w.size, step)
    return w, m, v


def inflight(replicas: Sequence[int], depth: int = 0) -> List[int]:
    R = np.ascontiguousarray(replicas, np.int32)
    k = np.zeros(len(R), np.int32)
    rc = lib().orc_inflight(_ptr(R), len(R), depth, _ptr(k))
    if rc != 0:
        raise ValueError("invalid depth override for a replicated plan")
    return [int(x) for x in k]


@dataclass
class RunResult:
    events: list          # tuples (worker, stage, replica, seq, kind, minibatch, vin, vout)
    times: np.ndarray     # [n_events, 2] start, end
    version_map: np.ndarray  # [n_stages, M]
    params: Optional[List[np.ndarray]]
    losses: np.ndarray
    makespan: float
    bubble: float
    max_live: np.ndarray = None  # [n_stages] widest weight-version window held (pin P10)


def run(layers, stage_last, replicas, B, M, params=None, data=None, optimizer=0, lr=0.05,
        beta1=0.9, beta2=0.999, eps=1e-8, depth=0, math=True, stash=True,
        fwd_time=None, bwd_time=None, vertical_sync=False, gpipe=False) -> RunResult:
    """Simulate PipeDream training.  ``params`` is a list of per-layer flat arrays.
    ``vertical_sync``: every stage uses the version the input stage tagged t with (§3.3).
    ``gpipe``: the §5.4 comparison schedule -- flush every D = ``depth`` (0 => n) minibatches,
    one update per group with the group's mean gradient (L1277-1279, R27)."""
    n = len(stage_last)
    lay = _layers(layers)
    sl = np.ascontiguousarray(stage_last, np.int32)
    rp = np.ascontiguousarray(replicas, np.int32)
    mode = (1 if math else 0) | (0 if stash else 2) | (4 if vertical_sync else 0) | (8 if gpipe else 0)
    inputs = tokens = labels = None
    n_data = 1
    if data is not None:
        inputs, tokens, labels = data
        n_data = (labels.shape[0])
        inputs = None if inputs is None else np.ascontiguousarray(inputs, np.float32)
        tokens = None if tokens is None else np.ascontiguousarray(tokens, np.int32)
        labels = np.ascontiguousarray(labels, np.int32)
    flat = None
    if math:
        flat = np.ascontiguousarray(np.concatenate([np.asarray(p, np.float32).ravel() for p in params]))
    cap = 3 * M * n + 16  # every stage runs F, B, U once per minibatch
    ev = (OrcEvent * cap)()
    nev = C.c_int(0)
    vmap = np.full((n, M), -1, np.int32)
    losses = np.zeros(M, np.float32)
    max_live = np.zeros(n, np.int32)
    mk = C.c_double(0)
    bub = C.c_double(0)
    ft = None if fwd_time is None else np.ascontiguousarray(fwd_time, np.float64)
    bt = None if bwd_time is None else np.ascontiguousarray(bwd_time, np.float64)
    rc = lib().orc_run(lay, len(layers), _ptr(sl), _ptr(rp), n, depth, B, M, optimizer, lr, beta1, beta2,
                       eps, mode, _ptr(inputs), _ptr(tokens), _ptr(labels), n_data, _ptr(flat), _ptr(ft),
                       _ptr(bt), ev, cap, C.byref(nev), _ptr(vmap), _ptr(losses), C.byref(mk), C.byref(bub),
                       _ptr(max_live))
    if rc == -2:
        raise RuntimeError("oracle: deadlock")
    if rc != 0:
        raise ValueError(f"oracle: orc_run returned {rc}")
    evs = [(e.worker, e.stage, e.replica, e.seq, chr(e.kind), e.minibatch, e.version_in, e.version_out)
           for e in ev[:nev.value]]
    times = np.array([(e.start, e.end) for e in ev[:nev.value]], np.float64).reshape(-1, 2)
    out_params = None
    if math:
        out_params, off = [], 0
        for L, p in zip(layers, params):
            k = np.asarray(p).size
            out_params.append(flat[off:off + k].copy())
            off += k
    return RunResult(evs, times, vmap, out_params, losses, mk.value, bub.value, max_live)


@dataclass
class Plan:
    stage_last: List[int]
    replicas: List[int]
    noam: int
    slowest: float


def plan(T, a, w, gpus, bandwidth=900e9, max_replicas=0, comm_model=0) -> Plan:
    T = np.ascontiguousarray(T, np.float64)
    a = np.ascontiguousarray(a, np.uint64)
    w = np.ascontiguousarray(w, np.uint64)
    N = len(T)
    ns = C.c_int(0)
    sl = np.zeros(N, np.int32)
    sr = np.zeros(N, np.int32)
    noam = C.c_int(0)
    slow = C.c_double(0)
    rc = lib().orc_plan(_ptr(T), _ptr(a), _ptr(w), N, gpus, bandwidth, max_replicas, comm_model,
                        C.byref(ns), _ptr(sl), _ptr(sr), C.byref(noam), C.byref(slow))
    if rc == -7:
        raise ValueError("infeasible")
    if rc != 0:
        raise ValueError(f"orc_plan returned {rc}")
    n = ns.value
    return Plan([int(x) for x in sl[:n]], [int(x) for x in sr[:n]], noam.value, slow.value)


def plan_levels(T, a, w, levels, max_replicas=0, comm_model=0) -> Plan:
    """Hierarchical §3.1 partitioner (Fig. 7): levels = [(m_1, B_1), ..., (m_L, B_L)], lowest
    level first; GPUs = prod m_k.  The plan comes back flattened (see oracle.cpp)."""
    T = np.ascontiguousarray(T, np.float64)
    a = np.ascontiguousarray(a, np.uint64)
    w = np.ascontiguousarray(w, np.uint64)
    N = len(T)
    lm = np.ascontiguousarray([m for m, _ in levels], np.int32)
    lb = np.ascontiguousarray([b for _, b in levels], np.float64)
    ns = C.c_int(0)
    sl = np.zeros(N, np.int32)
    sr = np.zeros(N, np.int32)
    noam = C.c_int(0)
    slow = C.c_double(0)
    rc = lib().orc_plan_levels(_ptr(T), _ptr(a), _ptr(w), N, len(levels), _ptr(lm), _ptr(lb), max_replicas, comm_model,
                               C.byref(ns), _ptr(sl), _ptr(sr), C.byref(noam), C.byref(slow))
    if rc == -7:
        raise ValueError("infeasible")
    if rc != 0:
        raise ValueError(f"orc_plan_levels returned {rc}")
    n = ns.value
    return Plan([int(x) for x in sl[:n]], [int(x) for x in sr[:n]], noam.value, slow.value)

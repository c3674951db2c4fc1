"""P1, P2, P7 and the negative controls: the oracle's pipelined training math against an
independent fp64 torch evaluation of the paper's update rules."""
import numpy as np
import pytest

import oracle
import synth
from synth import Layer, LINEAR, ACT_RELU
import torchref

TOL = 2e-4  # fp32 oracle vs fp64 torch, max relative error (R23)


def _delta_err(out, ref, init):
    """Relative error on parameter DELTAS (p_N - p_0), so version bugs are not hidden."""
    return torchref.delta_err(out, ref, init)


def _run(wl, stage_last, replicas, M, n_data, stash=True, depth=0):
    p0 = synth.init_params(wl.layers)
    data = synth.make_data(wl, n_data)
    r = oracle.run(wl.layers, stage_last, replicas, wl.batch, M, p0, data, wl.optimizer, wl.lr,
                   wl.beta1, wl.beta2, wl.eps, depth=depth, stash=stash)
    return p0, data, r


def _textbook_sgd(wl, p0, data, M, batch_of=lambda t: [t]):
    """Vanilla minibatch training (L1227-1231): w(t+1) = w(t) - lr * grad f(w(t))."""
    opt = torchref.Opt(wl.optimizer, wl.lr, wl.beta1, wl.beta2, wl.eps)
    ws = torchref.to_t(p0, wl.layers)
    flat = [t for ps in ws for t in ps]
    st = opt.make_state(flat)
    n_data = data[2].shape[0]
    for t in range(M):
        gsum = None
        for tt in batch_of(t):
            x, tk, lb = torchref.batch(data, tt % n_data)
            gs, _ = torchref.grads_at(wl.layers, wl.batch, ws, x, tk, lb)
            g = [gg for ps in gs for gg in ps]
            gsum = g if gsum is None else [a + b for a, b in zip(gsum, g)]
        k = len(batch_of(t))
        flat = opt.step(flat, [g / k for g in gsum], st)
        i, ws = 0, []
        for L in wl.layers:
            c = len(synth.param_shapes(L))
            ws.append(flat[i:i + c])
            i += c
    return [torchref.flat_of(ps) for ps in ws]


# ---------------- P1: one stage reduces to plain minibatch SGD ---------------

@pytest.mark.parametrize("name", ["mlp4096", "gnmt8", "vgg16"])
def test_single_stage_is_plain_sgd(name):
    wl = synth.workload(name, reduced=True)
    M = 4
    p0, data, r = _run(wl, [len(wl.layers) - 1], [1], M, n_data=3)
    ref = _textbook_sgd(wl, p0, data, M)
    assert _delta_err(r.params, ref, p0) < TOL
    assert list(r.version_map[0]) == list(range(M))


def test_single_stage_cfg1_full_size():
    wl = synth.workload("mlp_small")
    M = 8
    p0, data, r = _run(wl, [2], [1], M, n_data=8)
    ref = _textbook_sgd(wl, p0, data, M)
    assert _delta_err(r.params, ref, p0) < TOL


# ---------------- P2: weight-stashing update == L1233-1241 term by term ---------------

def _paper_versions(n):
    # straight pipeline: stage s (0-based) uses w_s^(t-n+s+1), clamped at 0 (L1237-1241, R5)
    return lambda s, t: max(0, t - n + s + 1)


CASES = [
    ("mlp_small", None, [1, 2], [1, 1], 8),          # cfg 1 at full size
    ("mlp4096", True, [3, 7, 11, 15], [1] * 4, 16),  # cfg 2 shape, width 64
    ("mlp4096", True, [0, 1, 2, 15], [1] * 4, 12),
    ("gnmt8", True, [4, 9], [1, 1], 8),              # cfg 3 2-stage, reduced
    ("gnmt8", True, [2, 5, 8, 9], [1] * 4, 12),      # cfg 3 4-stage, reduced
    ("vgg16", True, [2, 5], [1, 1], 6),              # VGG-like 2 stages
]


@pytest.mark.parametrize("name,reduced,last,reps,M", CASES)
def test_stashing_matches_staleness_formula(name, reduced, last, reps, M):
    wl = synth.workload(name, reduced=bool(reduced))
    p0, data, r = _run(wl, last, reps, M, n_data=5)
    opt = torchref.Opt(wl.optimizer, wl.lr, wl.beta1, wl.beta2, wl.eps)
    ref = torchref.staleness_evaluator(wl.layers, last, reps, wl.batch, M, p0, data,
                                       _paper_versions(len(last)), opt)
    assert _delta_err(r.params, ref, p0) < TOL


@pytest.mark.parametrize("reps", [[2, 1], [3, 1], [7, 1]])
def test_replicated_input_stage_matches_evaluator(reps):
    # replicated stages: v(s,t) = max(0, floor(t/R_s) - k_s + 1) (P6) and round means (R7)
    wl = synth.workload("mlp4096", reduced=True)
    last = [7, 15]
    M = 4 * reps[0]
    p0, data, r = _run(wl, last, reps, M, n_data=5)
    k = oracle.inflight(reps)
    opt = torchref.Opt(wl.optimizer, wl.lr)
    ref = torchref.staleness_evaluator(wl.layers, last, reps, wl.batch, M, p0, data,
                                       lambda s, t: max(0, t // reps[s] - k[s] + 1), opt)
    assert _delta_err(r.params, ref, p0) < TOL


# ---------------- P7: pure data parallelism == BSP / batch-R*B SGD ---------------

def test_pure_dp_is_bsp():
    wl = synth.workload("mlp4096", reduced=True)
    R, rounds = 4, 3
    M = R * rounds
    p0, data, r = _run(wl, [len(wl.layers) - 1], [R], M, n_data=M)
    assert list(r.version_map[0]) == [t // R for t in range(M)]
    ref = _textbook_sgd(wl, p0, data, rounds, batch_of=lambda j: list(range(j * R, j * R + R)))
    assert _delta_err(r.params, ref, p0) < TOL


# ---------------- negative controls (mutation tests for the tolerance) ---------------

def test_negative_control_no_stashing_fails_formula():
    wl = synth.workload("mlp4096", reduced=True)
    last, reps, M = [3, 7, 11, 15], [1] * 4, 16
    p0, data, r = _run(wl, last, reps, M, n_data=5, stash=False)
    opt = torchref.Opt(wl.optimizer, wl.lr)
    ref = torchref.staleness_evaluator(wl.layers, last, reps, wl.batch, M, p0, data, _paper_versions(4), opt)
    assert _delta_err(r.params, ref, p0) > 100 * TOL


def test_negative_control_off_by_one_version_fails():
    wl = synth.workload("mlp4096", reduced=True)
    last, reps, M = [3, 7, 11, 15], [1] * 4, 16
    p0, data, r = _run(wl, last, reps, M, n_data=5)
    opt = torchref.Opt(wl.optimizer, wl.lr)
    wrong = lambda s, t: max(0, t - 4 + s + 2) if s < 3 else t
    ref = torchref.staleness_evaluator(wl.layers, last, reps, wl.batch, M, p0, data, wrong, opt)
    assert _delta_err(r.params, ref, p0) > 100 * TOL


def test_depth_override_gives_model_parallel_semantics():
    # D = 1: one minibatch in flight => plain SGD regardless of the partition (Fig. 2)
    wl = synth.workload("mlp4096", reduced=True)
    M = 6
    p0, data, r = _run(wl, [3, 7, 11, 15], [1] * 4, M, n_data=3, depth=1)
    ref = _textbook_sgd(wl, p0, data, M)
    assert _delta_err(r.params, ref, p0) < TOL

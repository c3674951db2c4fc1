"""Vertical sync (§3.3 "Vertical Sync", L1175-1203) in the
oracle, pinned against the paper's update rule evaluated literally (L1247-1253):

    w(t+1) = w(t) - nu * grad f(w_1^(t-n+1), w_2^(t-n+1), ..., w_n^(t-n+1))

i.e. every stage computes minibatch t's gradient at the version the input stage tagged t with,
which for a straight pipeline of in-flight count k_0 is max(0, t - k_0 + 1) (= t - n + 1
clamped for the default k_0 = n, R25)."""
import numpy as np
import pytest

import oracle
import synth
import torchref

TOL = 2e-4  # fp32 oracle vs fp64 torch (R23), as for weight stashing


def _run(wl, last, M, n_data=5, vsync=True, depth=0):
    p0 = synth.init_params(wl.layers)
    data = synth.make_data(wl, n_data)
    r = oracle.run(wl.layers, last, [1] * len(last), wl.batch, M, p0, data, wl.optimizer, wl.lr,
                   wl.beta1, wl.beta2, wl.eps, depth=depth, vertical_sync=vsync)
    return p0, data, r


def _tag(k0):
    return lambda s, t: max(0, t - k0 + 1)


CASES = [
    ("mlp4096", [7, 15], 8),
    ("mlp4096", [3, 7, 11, 15], 16),
    ("mlp4096", [0, 1, 2, 15], 12),
    ("gnmt8", [4, 9], 8),
    ("gnmt8", [2, 5, 8, 9], 12),
    ("vgg16", [2, 5], 6),
]


@pytest.mark.parametrize("name,last,M", CASES)
def test_vertical_sync_matches_paper_formula(name, last, M):
    wl = synth.workload(name, reduced=True)
    p0, data, r = _run(wl, last, M)
    k0 = oracle.inflight([1] * len(last))[0]
    opt = torchref.Opt(wl.optimizer, wl.lr, wl.beta1, wl.beta2, wl.eps)
    ref = torchref.staleness_evaluator(wl.layers, last, [1] * len(last), wl.batch, M, p0, data, _tag(k0), opt)
    assert torchref.delta_err(r.params, ref, p0) < TOL


def test_vertical_sync_differs_from_weight_stashing():
    # negative control: the two rules differ on every stage but the first, so the vsync
    # oracle must NOT match the weight-stashing formula (and vice versa)
    wl = synth.workload("mlp4096", reduced=True)
    last = [3, 7, 11, 15]
    M = 16
    p0, data, r = _run(wl, last, M)
    opt = torchref.Opt(wl.optimizer, wl.lr)
    k = oracle.inflight([1] * 4)
    stash_ref = torchref.staleness_evaluator(wl.layers, last, [1] * 4, wl.batch, M, p0, data,
                                             lambda s, t: max(0, t - k[s] + 1), opt)
    assert torchref.delta_err(r.params, stash_ref, p0) > 100 * TOL
    # and the stashing oracle on the same inputs does match it
    _, _, r_stash = _run(wl, last, M, vsync=False)
    assert torchref.delta_err(r_stash.params, stash_ref, p0) < TOL


def test_vertical_sync_depth_override():
    # R19 depth D: k_0 = D, so every stage uses max(0, t - D + 1)
    wl = synth.workload("mlp4096", reduced=True)
    last = [3, 7, 11, 15]
    M, D = 12, 2
    p0, data, r = _run(wl, last, M, depth=D)
    assert (r.version_map == np.array([[max(0, t - D + 1) for t in range(M)]] * 4)).all()
    opt = torchref.Opt(wl.optimizer, wl.lr)
    ref = torchref.staleness_evaluator(wl.layers, last, [1] * 4, wl.batch, M, p0, data, _tag(D), opt)
    assert torchref.delta_err(r.params, ref, p0) < TOL


def test_single_stage_vertical_sync_is_plain_sgd():
    # one stage: the tag is the latest version, so vsync == stashing == textbook SGD (bit-exact)
    wl = synth.workload("mlp4096", reduced=True)
    _, _, a = _run(wl, [15], 6)
    _, _, b = _run(wl, [15], 6, vsync=False)
    for x, y in zip(a.params, b.params):
        assert np.array_equal(x, y)


@pytest.mark.parametrize("n", [2, 4, 8])
def test_vertical_sync_trace(n):
    wl = synth.workload("mlp4096", reduced=True)
    per = 16 // n
    last = [per * (s + 1) - 1 for s in range(n)]
    M = 3 * n
    r = oracle.run(wl.layers, last, [1] * n, wl.batch, M, math=False, vertical_sync=True)
    k0 = n
    tags = [max(0, t - k0 + 1) for t in range(M)]
    # version map: every stage uses the input stage's tag (L1180-1186)
    assert (r.version_map == np.array([tags] * n)).all()
    # the op order is the weight-stashing schedule's (vertical sync changes versions only)
    rs = oracle.run(wl.layers, last, [1] * n, wl.batch, M, math=False)
    assert [e[:6] for e in r.events] == [e[:6] for e in rs.events]
    for e in r.events:
        w, s, rep, seq, kind, t, vin, vout = e
        if kind in "FB":
            assert vin == vout == tags[t]
        else:
            assert vout == vin + 1
    # each worker's updates count 0, 1, 2, ...
    for s in range(n):
        us = [e for e in r.events if e[1] == s and e[4] == "U"]
        assert [e[6] for e in us] == list(range(M))


def _needed_window(events, stage):
    """Widest window of weight versions worker `stage` must hold after any of its updates: the
    latest version and every version a later F or B of this worker reads (from the trace)."""
    ops = [e for e in events if e[1] == stage]
    widest = 1
    for i, e in enumerate(ops):
        if e[4] != "U":
            continue
        latest = e[7]
        later = [x[6] for x in ops[i + 1:] if x[4] in "FB"]
        lo = min(later + [latest])
        widest = max(widest, latest - lo + 1)
    return widest


@pytest.mark.parametrize("n", [2, 4, 8])
def test_stash_ring_depth(n):
    """P10 for both rules, read off the trace: weight stashing needs k_s versions at stage s;
    vertical sync needs k_0 at EVERY stage -- the ring depth the runtime allocates (R25)."""
    wl = synth.workload("mlp4096", reduced=True)
    per = 16 // n
    last = [per * (s + 1) - 1 for s in range(n)]
    M = 4 * n
    k = oracle.inflight([1] * n)
    rs = oracle.run(wl.layers, last, [1] * n, wl.batch, M, math=False)
    rv = oracle.run(wl.layers, last, [1] * n, wl.batch, M, math=False, vertical_sync=True)
    for s in range(n):
        assert _needed_window(rs.events, s) == k[s]
        assert rs.max_live[s] == k[s]
        assert _needed_window(rv.events, s) == k[0]


def test_vertical_sync_rejects_replicated_plans():
    wl = synth.workload("mlp4096", reduced=True)
    with pytest.raises(ValueError):
        oracle.run(wl.layers, [7, 15], [2, 1], wl.batch, 4, math=False, vertical_sync=True)

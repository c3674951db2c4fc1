"""GPipe-style flush schedule with gradient aggregation in the oracle (
PAPER.md §5.4 "Comparison to Inter-batch Parallelism", gradient aggregation
L1277-1279; R27), pinned against what the paper and the mathematics fix:

* every minibatch of flush group g = floor(t / D) runs F and B with the same version g, and
  one update per group applies the group's mean gradient:
      w_{g+1} = w_g - nu * (1/D) sum_{t in group g} grad f_t(w_g)
  evaluated literally in torch fp64 autograd (a different implementation of the layer math);
* that update is one SGD step on the D*B samples of the group (the loss is a per-sample
  mean), checked against the oracle's single-stage plain-SGD path (pinned to torch by P1)
  fed the concatenated minibatches;
* the static op lists (F^D B^D U per group; the last stage F B back to back), the version
  map t -> floor(t / D) and the update events, from the schedule alone."""
import numpy as np
import pytest

import oracle
import synth
import torchref

TOL = 2e-4  # fp32 oracle vs fp64 torch (R23), as for the other training pins


def _group_sgd_ref(wl, last, M, D, p0, data):
    """PAPER.md L1277-1279 + §5.4 literally: per group, full-model gradients of every
    minibatch at the group's weights, added in t order, times 1/D, one optimizer step."""
    import torch
    opt = torchref.Opt(wl.optimizer, wl.lr, wl.beta1, wl.beta2, wl.eps)
    w = torchref.to_t(p0, wl.layers)
    flat = [t for ps in w for t in ps]
    st = opt.make_state(flat)
    n_data = data[2].shape[0]
    for g in range(M // D):
        acc = None
        for t in range(g * D, (g + 1) * D):
            x, tk, lb = torchref.batch(data, t % n_data)
            gs, _ = torchref.grads_at(wl.layers, wl.batch, w, x, tk, lb)
            gf = [x for ps in gs for x in ps]
            acc = gf if acc is None else [a + b for a, b in zip(acc, gf)]
        acc = [a / D for a in acc]
        flat = opt.step(flat, acc, st)
        w, i = [], 0
        for L in wl.layers:
            k = len(synth.param_shapes(L))
            w.append(flat[i:i + k])
            i += k
    del torch
    return [torchref.flat_of(ps) for ps in w]


CASES = [
    ("mlp4096", [7, 15], 8, 2),
    ("mlp4096", [3, 7, 11, 15], 16, 4),
    ("mlp4096", [3, 7, 11, 15], 12, 3),
    ("gnmt8", [4, 9], 8, 2),
    ("gnmt8", [2, 5, 8, 9], 16, 4),
    ("vgg16", [2, 5], 6, 3),
]


@pytest.mark.parametrize("name,last,M,D", CASES)
def test_gpipe_matches_group_mean_update(name, last, M, D):
    wl = synth.workload(name, reduced=True)
    p0 = synth.init_params(wl.layers)
    data = synth.make_data(wl, 5)
    r = oracle.run(wl.layers, last, [1] * len(last), wl.batch, M, p0, data, wl.optimizer, wl.lr,
                   wl.beta1, wl.beta2, wl.eps, depth=D, gpipe=True)
    ref = _group_sgd_ref(wl, last, M, D, p0, data)
    assert torchref.delta_err(r.params, ref, p0) < TOL


def test_gpipe_is_one_sgd_step_on_the_concatenated_group():
    # MLP: softmax-CE is a mean over rows, so the mean of D minibatch gradients is the
    # gradient of the mean over the D*B samples: GPipe on 4 stages == one stage, batch D*B
    wl = synth.workload("mlp4096", reduced=True)
    last, D, G = [3, 7, 11, 15], 4, 3
    p0 = synth.init_params(wl.layers)
    inputs, tokens, labels = synth.make_data(wl, D * G)
    r = oracle.run(wl.layers, last, [1] * 4, wl.batch, D * G, p0, (inputs, tokens, labels), wl.optimizer,
                   wl.lr, depth=D, gpipe=True)
    big_in = inputs.reshape(G, D * inputs.shape[1])
    big_lb = labels.reshape(G, D * labels.shape[1])
    single = oracle.run(wl.layers, [15], [1], wl.batch * D, G, p0, (big_in, None, big_lb), wl.optimizer, wl.lr)
    assert torchref.delta_err(r.params, single.params, p0) < TOL


def test_gpipe_differs_from_weight_stashing():
    wl = synth.workload("mlp4096", reduced=True)
    last, M = [3, 7, 11, 15], 16
    p0 = synth.init_params(wl.layers)
    data = synth.make_data(wl, 5)
    a = oracle.run(wl.layers, last, [1] * 4, wl.batch, M, p0, data, wl.optimizer, wl.lr, gpipe=True)
    b = oracle.run(wl.layers, last, [1] * 4, wl.batch, M, p0, data, wl.optimizer, wl.lr)
    ref = _group_sgd_ref(wl, last, M, 4, p0, data)
    assert torchref.delta_err(a.params, ref, p0) < TOL
    assert torchref.delta_err(b.params, ref, p0) > 100 * TOL


def _expected_ops(n, s, M, D):
    ops = []
    for g in range(M // D):
        ts = range(g * D, (g + 1) * D)
        if s + 1 < n:
            ops += [("F", t, g, g) for t in ts] + [("B", t, g, g) for t in ts]
        else:
            for t in ts:
                ops += [("F", t, g, g), ("B", t, g, g)]
        ops.append(("U", g, g, g + 1))
    return ops


@pytest.mark.parametrize("n,D,M", [(2, 2, 8), (4, 4, 8), (4, 2, 8), (8, 8, 16), (3, 5, 10), (1, 3, 6)])
def test_gpipe_schedule(n, D, M):
    wl = synth.workload("mlp4096", reduced=True)
    per = 16 // n
    last = [per * (s + 1) - 1 for s in range(n)]
    last[-1] = 15
    r = oracle.run(wl.layers, last, [1] * n, wl.batch, M, math=False, depth=D, gpipe=True)
    for s in range(n):
        got = [(e[4], e[5], e[6], e[7]) for e in r.events if e[1] == s]
        assert got == _expected_ops(n, s, M, D)
    assert (r.version_map == np.array([[t // D for t in range(M)]] * n)).all()


def test_gpipe_default_depth_is_noam():
    # depth 0: the paper's "pipeline depth equivalent to NOAM" (L1955-1958): D = n
    wl = synth.workload("mlp4096", reduced=True)
    r = oracle.run(wl.layers, [3, 7, 11, 15], [1] * 4, wl.batch, 8, math=False, gpipe=True)
    assert (r.version_map == np.array([[t // 4 for t in range(8)]] * 4)).all()


def test_gpipe_flush_bubble():
    # unit F and B times: a flush every D minibatches idles every stage for the fill and the
    # drain of each group, so GPipe's bubble exceeds 1F1B's (which drains once), §5.4
    wl = synth.workload("mlp4096", reduced=True)
    n, M = 4, 32
    last = [3, 7, 11, 15]
    ft, bt = np.ones(n), 2 * np.ones(n)
    g = oracle.run(wl.layers, last, [1] * n, wl.batch, M, math=False, gpipe=True, fwd_time=ft, bwd_time=bt)
    p = oracle.run(wl.layers, last, [1] * n, wl.batch, M, math=False, fwd_time=ft, bwd_time=bt)
    assert g.bubble > p.bubble + 0.2
    # 1F1B: one fill + drain over M minibatches, (n-1)/(M+n-1)
    assert abs(p.bubble - (n - 1) / (M + n - 1)) < 1e-9


def test_gpipe_rejects_invalid():
    wl = synth.workload("mlp4096", reduced=True)
    with pytest.raises(ValueError):  # replicated stage
        oracle.run(wl.layers, [7, 15], [2, 1], wl.batch, 8, math=False, gpipe=True)
    with pytest.raises(ValueError):  # M not a multiple of D
        oracle.run(wl.layers, [7, 15], [1, 1], wl.batch, 7, math=False, depth=2, gpipe=True)
    with pytest.raises(ValueError):  # with vertical sync
        oracle.run(wl.layers, [7, 15], [1, 1], wl.batch, 8, math=False, gpipe=True, vertical_sync=True)

"""P9: the oracle's layer math against independent library routines (torch fp64 autograd,
numpy) at tiny shapes.  A dropped term, wrong sign/index or transposed operand in any
oracle layer fails one of these."""
import numpy as np
import pytest
import torch

import oracle
import synth
from synth import Layer, LINEAR, LSTM, CONV3X3, MAXPOOL2, EMBEDDING, ACT_RELU, ACT_NONE
import torchref

RTOL = 2e-5  # fp32 oracle vs fp64 reference, relative to the tensor's max magnitude


def _rel(a, b):
    b = np.asarray(b, np.float64)
    return float(np.abs(np.asarray(a, np.float64) - b).max() / max(np.abs(b).max(), 1e-30))


def _check_layer(L, B, seed=0, tokens=None):
    rng = np.random.default_rng(seed)
    p = synth.init_params([L], seed=seed)[0]
    if L.kind == EMBEDDING:
        x = None
    else:
        x = rng.standard_normal(oracle.in_size(L, B)).astype(np.float32)
    y = oracle.layer_forward(L, B, p, x, tokens)
    dy = rng.standard_normal(y.size).astype(np.float32)
    dx, dp = oracle.layer_backward(L, B, p, x, tokens, dy, need_dx=L.kind != EMBEDDING)

    ps = torchref.split_params(L, p)
    for t in ps:
        t.requires_grad_(True)
    xt = None if x is None else torch.tensor(x, dtype=torch.float64, requires_grad=True)
    tk = None if tokens is None else torch.tensor(tokens)
    yt = torchref.layer_forward(L, B, ps, xt, tk)
    assert _rel(y, yt.detach().numpy()) < RTOL
    (yt * torch.tensor(dy, dtype=torch.float64)).sum().backward()
    if ps:
        assert _rel(dp, torchref.flat_of([t.grad for t in ps])) < RTOL
    if xt is not None:
        assert _rel(dx, xt.grad.numpy()) < RTOL
    return y


@pytest.mark.parametrize("act", [ACT_NONE, ACT_RELU])
def test_linear(act):
    _check_layer(Layer(LINEAR, 13, 7, act), 5)


def test_linear_matches_numpy_matmul():
    L = Layer(LINEAR, 9, 4, ACT_NONE)
    rng = np.random.default_rng(3)
    p = synth.init_params([L], seed=3)[0]
    x = rng.standard_normal(6 * 9).astype(np.float32)
    y = oracle.layer_forward(L, 6, p, x)
    W, b = p[:36].reshape(4, 9), p[36:]
    ref = x.reshape(6, 9).astype(np.float64) @ W.T.astype(np.float64) + b
    assert _rel(y, ref.ravel()) < RTOL


def test_linear_per_token():
    _check_layer(Layer(LINEAR, 6, 5, ACT_NONE, seq_len=3), 2)


def test_lstm():
    _check_layer(Layer(LSTM, 5, 4, seq_len=4), 3)


def test_lstm_in_ne_hidden():
    _check_layer(Layer(LSTM, 7, 3, seq_len=3), 2, seed=5)


@pytest.mark.parametrize("act", [ACT_NONE, ACT_RELU])
def test_conv3x3(act):
    _check_layer(Layer(CONV3X3, 3, 4, act, height=5, width=6), 2)


def test_maxpool2():
    _check_layer(Layer(MAXPOOL2, 3, 3, height=4, width=6), 2)


def test_embedding():
    L = Layer(EMBEDDING, 11, 4, seq_len=3)
    tokens = np.random.default_rng(1).integers(0, 11, 3 * 2).astype(np.int32)
    tokens[1] = tokens[4]  # a repeated token exercises the scatter-add
    _check_layer(L, 2, tokens=tokens)


def test_softmax_ce_matches_torch():
    rng = np.random.default_rng(2)
    z = rng.standard_normal((7, 5)).astype(np.float32) * 3
    lab = rng.integers(0, 5, 7).astype(np.int32)
    loss, dz = oracle.softmax_ce(z, lab)
    zt = torch.tensor(z, dtype=torch.float64, requires_grad=True)
    lt = torch.nn.functional.cross_entropy(zt, torch.tensor(lab).long())
    lt.backward()
    assert abs(loss - lt.item()) < 1e-5
    assert _rel(dz, zt.grad.numpy()) < RTOL


def test_softmax_ce_uniform_closed_form():
    # all-equal logits: loss = log C exactly, dz = (1/C - onehot)/R
    z = np.zeros((4, 8), np.float32)
    lab = np.array([0, 3, 7, 1], np.int32)
    loss, dz = oracle.softmax_ce(z, lab)
    assert abs(loss - np.log(8)) < 1e-6
    ref = (np.full((4, 8), 1 / 8) - np.eye(8)[lab]) / 4
    assert np.abs(dz - ref).max() < 1e-7


def test_sgd_and_adam_update_closed_form():
    w = np.array([1.0, -2.0, 0.5], np.float32)
    g = np.array([0.1, 0.2, -0.3], np.float32)
    w1, _, _ = oracle.update(synth.SGD, 0.5, w, g)
    assert np.allclose(w1, w - 0.5 * g, atol=0)
    # Adam first step: m_hat = g, v_hat = g^2 => w - lr * g / (|g| + eps)
    w2, m, v = oracle.update(synth.ADAM, 0.01, w, g, step=1)
    assert np.allclose(w2, w - 0.01 * g / (np.abs(g) + 1e-8), rtol=1e-6)
    # second step against torch.optim.Adam
    wt = torch.tensor(w, dtype=torch.float64, requires_grad=True)
    opt = torch.optim.Adam([wt], lr=0.01, betas=(0.9, 0.999), eps=1e-8)
    for gg in (g, 2 * g):
        wt.grad = torch.tensor(gg, dtype=torch.float64)
        opt.step()
    w3, _, _ = oracle.update(synth.ADAM, 0.01, w2, 2 * g, m, v, step=2)
    assert np.abs(w3 - wt.detach().numpy()).max() < 1e-6

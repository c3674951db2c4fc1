"""Independent fp64 reference built from torch library routines (F.linear, nn.LSTM, F.conv2d,
F.max_pool2d, F.embedding, F.cross_entropy, autograd).  Used only to PIN the oracle
(tests/test_oracle_*.py): it shares no code with oracle/oracle.cpp.
"""
from __future__ import annotations

import numpy as np
import torch
import torch.nn.functional as F

import synth
from synth import LINEAR, LSTM, CONV3X3, MAXPOOL2, EMBEDDING, ACT_RELU

DT = torch.float64


def split_params(L, flat):
    """flat per-layer array -> list of torch tensors in the layout of synth.param_shapes."""
    out, off = [], 0
    for shp in synth.param_shapes(L):
        n = int(np.prod(shp))
        out.append(torch.tensor(np.asarray(flat[off:off + n]), dtype=DT).reshape(shp))
        off += n
    return out


def layer_forward(L, B, ps, x=None, tokens=None):
    """x is a flat fp64 tensor in the repo's activation layout; returns flat output."""
    if L.kind == LINEAR:
        R = B * (L.seq_len if L.seq_len else 1)
        y = F.linear(x.reshape(R, L.in_), ps[0], ps[1])
        if L.act == ACT_RELU:
            y = torch.relu(y)
        return y.reshape(-1)
    if L.kind == LSTM:
        lstm = torch.nn.LSTM(L.in_, L.out).to(DT)
        with torch.no_grad():
            pass
        # functional call with our tensors (keeps autograd to ps)
        params = {"weight_ih_l0": ps[0], "weight_hh_l0": ps[1], "bias_ih_l0": ps[2], "bias_hh_l0": ps[3]}
        y, _ = torch.func.functional_call(lstm, params, (x.reshape(L.seq_len, B, L.in_),))
        return y.reshape(-1)
    if L.kind == CONV3X3:
        xi = x.reshape(B, L.height, L.width, L.in_).permute(0, 3, 1, 2)
        y = F.conv2d(xi, ps[0], ps[1], padding=1)
        if L.act == ACT_RELU:
            y = torch.relu(y)
        return y.permute(0, 2, 3, 1).reshape(-1)
    if L.kind == MAXPOOL2:
        xi = x.reshape(B, L.height, L.width, L.in_).permute(0, 3, 1, 2)
        y = F.max_pool2d(xi, 2)
        return y.permute(0, 2, 3, 1).reshape(-1)
    if L.kind == EMBEDDING:
        return F.embedding(tokens.long(), ps[0]).reshape(-1)
    raise ValueError(L.kind)


def model_loss(layers, B, params_t, x=None, tokens=None, labels=None):
    """Full-model mean softmax-CE loss.  params_t: list (per layer) of lists of tensors."""
    h = x
    for L, ps in zip(layers, params_t):
        h = layer_forward(L, B, ps, h, tokens)
    last = layers[-1]
    logits = h.reshape(-1, last.out)
    return F.cross_entropy(logits, labels.long())


def to_t(flat_params, layers, requires_grad=False):
    out = []
    for L, p in zip(layers, flat_params):
        ts = split_params(L, p)
        for t in ts:
            t.requires_grad_(requires_grad)
        out.append(ts)
    return out


def flat_of(ts):
    if not ts:
        return np.zeros(0)
    return torch.cat([t.detach().reshape(-1) for t in ts]).numpy()


def batch(data, d):
    inputs, tokens, labels = data
    x = None if inputs is None else torch.tensor(inputs[d], dtype=DT)
    tk = None if tokens is None else torch.tensor(tokens[d])
    lb = torch.tensor(labels[d])
    return x, tk, lb


def grads_at(layers, B, stage_params_t, x, tk, lb):
    """Gradient of the full-model loss w.r.t. every layer's params at the given weights."""
    ts = [[t.detach().clone().requires_grad_(True) for t in ps] for ps in stage_params_t]
    loss = model_loss(layers, B, ts, x, tk, lb)
    flat = [t for ps in ts for t in ps]
    gs = torch.autograd.grad(loss, flat, allow_unused=True)
    out, i = [], 0
    for ps in ts:
        g = []
        for t in ps:
            g.append(torch.zeros_like(t) if gs[i] is None else gs[i])
            i += 1
        out.append(g)
    return out, float(loss.detach())


class Opt:
    """SGD / Adam on a list of tensors (textbook formulas; Adam as torch.optim.Adam)."""

    def __init__(self, kind, lr, b1=0.9, b2=0.999, eps=1e-8):
        self.kind, self.lr, self.b1, self.b2, self.eps = kind, lr, b1, b2, eps

    def make_state(self, ts):
        return {"step": 0, "m": [torch.zeros_like(t) for t in ts], "v": [torch.zeros_like(t) for t in ts]}

    def step(self, ts, gs, st):
        st["step"] += 1
        k = st["step"]
        new = []
        for i, (w, g) in enumerate(zip(ts, gs)):
            if self.kind == synth.SGD:
                new.append(w - self.lr * g)
            else:
                st["m"][i] = self.b1 * st["m"][i] + (1 - self.b1) * g
                st["v"][i] = self.b2 * st["v"][i] + (1 - self.b2) * g * g
                mh = st["m"][i] / (1 - self.b1 ** k)
                vh = st["v"][i] / (1 - self.b2 ** k)
                new.append(w - self.lr * mh / (torch.sqrt(vh) + self.eps))
        return new


def staleness_evaluator(layers, stage_last, replicas, B, M, params, data, version_fn, opt: Opt):
    """PAPER.md L1233-1241 evaluated literally (non-pipelined): for each minibatch t the
    full-model gradient is taken at the mixed vector (w_1^{v(0,t)}, ..., w_n^{v(n-1,t)}) and
    stage s's update is applied to its LATEST weights.  Replicated stages (R_s > 1) average
    the gradients of round j = {t : floor(t/R_s) = j} (L1345-1347).  ``version_fn(s, t)``
    gives v(s, t).  Returns final per-layer flat params."""
    n = len(stage_last)
    first = [0] + [x + 1 for x in stage_last[:-1]]
    stage_layers = [list(range(first[s], stage_last[s] + 1)) for s in range(n)]
    init = to_t(params, layers)
    hist = [[[t for l in stage_layers[s] for t in init[l]]] for s in range(n)]
    states = [opt.make_state(hist[s][0]) for s in range(n)]
    pending = [dict() for _ in range(n)]
    n_data = data[2].shape[0]
    for t in range(M):
        mixed = []
        for s in range(n):
            ws = hist[s][version_fn(s, t)]
            i = 0
            for l in stage_layers[s]:
                k = len(synth.param_shapes(layers[l]))
                mixed.append(ws[i:i + k])
                i += k
        x, tk, lb = batch(data, t % n_data)
        gs, _ = grads_at(layers, B, mixed, x, tk, lb)
        for s in range(n):
            g = [gg for l in stage_layers[s] for gg in gs[l]]
            j = t // replicas[s]
            pending[s].setdefault(j, []).append(g)
            if len(pending[s][j]) == replicas[s]:
                # mean = (sum in replica order) / R
                acc = [sum(gr[i] for gr in pending[s][j]) / replicas[s] for i in range(len(g))]
                hist[s].append(opt.step(hist[s][-1], acc, states[s]))
                del pending[s][j]
    out = []
    for s in range(n):
        ws, i = hist[s][-1], 0
        for l in stage_layers[s]:
            k = len(synth.param_shapes(layers[l]))
            out.append(flat_of(ws[i:i + k]))
            i += k
    return out


def delta_err(out, ref, init, floor=1e-2):
    """DESIGN.md R23 on parameter DELTAS: per tensor ||d_out - d_ref||_inf /
    max(||d_ref||_inf, floor * ||p_ref||_inf), max over tensors.  The floor keeps tensors
    whose total change is below fp32 resolution of the weights (vanishing gradients in deep
    uniform-init stacks) from dividing rounding noise by ~0."""
    worst = 0.0
    for o, r, i in zip(out, ref, init):
        o, r, i = (np.asarray(x, np.float64) for x in (o, r, i))
        if r.size == 0:
            continue
        den = max(np.abs(r - i).max(), floor * np.abs(r).max(), 1e-30)
        worst = max(worst, float(np.abs((o - i) - (r - i)).max() / den))
    return worst


def max_rel_err(a_list, b_list):
    """DESIGN.md R23: per tensor ||a-b||_inf / ||b||_inf, max over tensors."""
    worst = 0.0
    for a, b in zip(a_list, b_list):
        a = np.asarray(a, np.float64)
        b = np.asarray(b, np.float64)
        if b.size == 0:
            continue
        den = max(np.abs(b).max(), 1e-30)
        worst = max(worst, float(np.abs(a - b).max() / den))
    return worst

#!/usr/bin/env python
"""Where the bf16 path's tolerance comes from (tests/test_gpu_fullsize.py): one SGD step of a
full-size case (tests/fullsize_cases.py) in torch fp64 on the CPU, once exact and once with
bf16 rounding at the points where the CUDA path stores bf16 (weights, layer outputs, logits,
dlogits, input gradients; fp32/fp64 accumulation everywhere else).  Prints, per parameter
tensor, the max-norm relative gradient error bf16 rounding alone causes -- the floor any
correct bf16 implementation sits on.  Test infrastructure only (no oracle, no product code).
    python tools/bf16_emulate.py longk_dw vgg_conv1
"""
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
sys.path.insert(0, os.path.join(ROOT, "tests"))

import numpy as np  # noqa: E402
import torch  # noqa: E402
import torch.nn.functional as F  # noqa: E402

import synth  # noqa: E402
import fullsize_cases as fc  # noqa: E402

D = torch.float64


def bf(t):
    return t.to(torch.bfloat16).to(D)


def grads(name, q):
    wl = fc.workload(name)
    p0 = synth.init_params(wl.layers)
    x, _, lab = synth.make_data(wl, 1)
    if name == "longk_dw":
        R = wl.batch * 50
        X = torch.tensor(x[0], dtype=D).reshape(R, 256)
        y = torch.tensor(lab[0]).long()
        W0 = torch.tensor(p0[0][:65536], dtype=D).reshape(256, 256)
        b0 = torch.tensor(p0[0][65536:], dtype=D)
        W1 = torch.tensor(p0[1][:65536], dtype=D).reshape(256, 256)
        b1 = torch.tensor(p0[1][65536:], dtype=D)
        Xq, W0q, W1q = q(X), q(W0), q(W1)
        h = q(torch.relu(Xq @ W0q.T + b0))
        z = q(h @ W1q.T + b1)
        p = torch.softmax(z, 1)
        d = p.clone()
        d[torch.arange(R), y] -= 1
        d = q(d / R)
        dh = q((d @ W1q) * (h > 0))
        return {"0_0": dh.T @ Xq, "0_1": dh.sum(0), "1_0": d.T @ h, "1_1": d.sum(0)}
    if name == "vgg_conv1":
        X = torch.tensor(x[0], dtype=D).reshape(1, 224, 224, 3).permute(0, 3, 1, 2)
        y = torch.tensor(lab[0]).long()
        Wc = torch.tensor(p0[0][:64 * 27], dtype=D).reshape(64, 3, 3, 3)
        bc = torch.tensor(p0[0][64 * 27:], dtype=D)
        Wf = torch.tensor(p0[2][:16 * 802816], dtype=D).reshape(16, 802816)
        bfc = torch.tensor(p0[2][16 * 802816:], dtype=D)
        Xq, Wcq, Wfq = q(X), q(Wc), q(Wf)
        a = q(torch.relu(F.conv2d(Xq, Wcq, bc, padding=1)))          # conv output, NCHW
        pool, idx = F.max_pool2d(a, 2, return_indices=True)           # exact (a selection)
        flat = pool.permute(0, 2, 3, 1).reshape(1, -1)                # NHWC flatten
        z = q(flat @ Wfq.T + bfc)
        p = torch.softmax(z, 1)
        d = p.clone()
        d[0, y] -= 1
        d = q(d)
        dflat = q(d @ Wfq)
        dpool = dflat.reshape(1, 112, 112, 64).permute(0, 3, 1, 2)
        da = F.max_unpool2d(dpool, idx, 2, output_size=a.shape[2:]) * (a > 0)
        da = q(da)
        dWc = torch.nn.grad.conv2d_weight(Xq, Wc.shape, da, padding=1)
        return {"0_0": dWc, "0_1": da.sum((0, 2, 3)), "2_0": d.T @ flat, "2_1": d.sum(0)}
    raise KeyError(name)


if __name__ == "__main__":
    for name in sys.argv[1:]:
        ex, bq = grads(name, lambda t: t), grads(name, bf)
        for k in ex:
            e = float((bq[k] - ex[k]).abs().max() / ex[k].abs().max())
            print(f"{name} tensor {k}: bf16-rounding gradient error {e:.4f}")

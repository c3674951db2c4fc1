"""Parity cases at the sizes the bench runs (VERDICT r1 "next round" #2).

Each case is one pd_run of a single stage (plain SGD, k = 1: F, B, U of one minibatch,
PAPER.md L1225-1231) through exactly the kernel path the full-size bench takes:

  gnmt16_wave   Emb(512, 1024) -> 16 x LSTM(1024), T = 4, B = 64 -> Linear(1024, 512) -> CE:
                the 16-layer wavefront (lstm_wave.cu) with its L2-residency split, the
                long-K (T*B rows) 2-CTA weight-gradient GEMMs, the fused bias updates.
                The oracle needs ~8 min single-threaded for it, so its expected values are
                computed once by tests/gen_golden_fullsize.py (which calls only oracle/ and
                synth/) and stored, sampled, under tests/golden/.
  longk_dw      Linear(256, 256)+ReLU -> Linear(256, 256) applied per token over T = 50,
                B = 64 (K = T*B = 3200 rows): the default long-K weight-gradient path
                (2-CTA GEMM -> fp32 gradient -> vectorised SGD), no knobs.
  vgg_conv1     conv3x3(3 -> 64) on 224 x 224, B = 1 -> maxpool -> Linear(112*112*64, 16):
                the packed-tap (9 taps x 8 channels = one K-block) conv1 forward and weight
                gradient at VGG-16's input size.

The sampled comparison: parameter deltas p_1 - p_0 at `SAMPLES` seeded positions per tensor
plus the positions of the tensor's largest oracle deltas, error per tensor = max |d_gpu -
d_ref| / max(max |d_ref| over the WHOLE tensor, 1e-2 max |p_ref|) (R23).
"""
from __future__ import annotations

import numpy as np

import synth

SAMPLES = 4096
TOP = 256
LR = 1.0  # one SGD step: the delta IS -lr * gradient, at a size bf16 resolves


def case(name):
    """(layers, B, lr) of a full-size case."""
    if name == "gnmt16_wave":
        return synth.gnmt(16, 1024, 512, 4, 64), 64, LR
    if name == "longk_dw":
        layers = [synth.Layer(synth.LINEAR, 256, 256, synth.ACT_RELU, seq_len=50),
                  synth.Layer(synth.LINEAR, 256, 256, synth.ACT_NONE, seq_len=50)]
        return layers, 64, 0.5
    if name == "vgg_conv1":
        layers = [synth.Layer(synth.CONV3X3, 3, 64, synth.ACT_RELU, height=224, width=224),
                  synth.Layer(synth.MAXPOOL2, 64, 64, height=224, width=224),
                  synth.Layer(synth.LINEAR, 112 * 112 * 64, 16)]
        return layers, 1, 0.05
    raise KeyError(name)


def workload(name):
    layers, B, lr = case(name)
    return synth.Workload(name, layers, B, synth.SGD, lr)


def tensor_slices(layers):
    """(layer, name, start, stop) of every parameter tensor in each layer's flat array."""
    out = []
    for l, L in enumerate(layers):
        off = 0
        for k, shp in enumerate(synth.param_shapes(L)):
            n = int(np.prod(shp))
            out.append((l, k, off, off + n))
            off += n
    return out


def sample_positions(ref_delta, n, seed):
    """Seeded uniform positions plus the largest |delta| positions of one tensor."""
    rng = np.random.default_rng(seed)
    pos = rng.integers(0, n, size=min(SAMPLES, n))
    top = np.argsort(-np.abs(ref_delta))[:TOP]
    return np.unique(np.concatenate([pos, top]))


def sampled_errors(golden, got):
    """Per-tensor floored delta errors of `got` (per-layer flat arrays) against a golden dict."""
    errs = {}
    for key in golden["keys"]:
        l, k = (int(x) for x in key.split("_"))
        start = int(golden[f"{key}_start"])
        pos = golden[f"{key}_pos"]
        d_ref = golden[f"{key}_dref"]
        p0 = golden[f"{key}_p0"]
        d_got = got[l][start + pos].astype(np.float64) - p0
        den = max(float(golden[f"{key}_dmax"]), 1e-2 * float(golden[f"{key}_pmax"]), 1e-30)
        errs[key] = float(np.abs(d_got - d_ref).max() / den)
    return errs

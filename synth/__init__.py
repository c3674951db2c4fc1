"""Seeded synthetic workloads shared by the oracle tests, the GPU parity tests and bench.py.

This module holds NO arithmetic of the method (no layer math, no schedule, no planner):
only workload *descriptions* (layer shapes of the BASELINE.json configs) and seeded
random inputs / initial weights.  Recipe:

* numpy ``default_rng``; data seed 1234, weight seed 42;
* dense inputs N(0, 1) fp32; class labels U{0..C-1}; tokens U{0..V-1}, labels are
  independent tokens;
* weights and biases U(-1/sqrt(fan_in), +1/sqrt(fan_in)); LSTM fan_in = H; embedding
  N(0, 1) (PyTorch's default, the embedding has no fan-in);
* parameter layout per layer (the parity contract): Linear W[out][in], b[out];
  LSTM W_ih[4H][in], W_hh[4H][H], b_ih[4H], b_hh[4H] (gates i, f, g, o);
  Conv W[Cout][Cin][3][3], b[Cout]; Embedding E[V][H]; MaxPool none.
* activations: rows are samples ([B][feat]); sequence models are time-major
  ([T][B][feat], tokens/labels [T][B]); images are NHWC.
"""
from __future__ import annotations

from dataclasses import dataclass, field
from typing import List, Optional

import numpy as np

LINEAR, LSTM, CONV3X3, MAXPOOL2, EMBEDDING = 0, 1, 2, 3, 4
ACT_NONE, ACT_RELU = 0, 1
SGD, ADAM = 0, 1

DATA_SEED = 1234
WEIGHT_SEED = 42


@dataclass(frozen=True)
class Layer:
    kind: int
    in_: int
    out: int
    act: int = ACT_NONE
    seq_len: int = 0
    height: int = 0
    width: int = 0

    def as_tuple(self):
        return (self.kind, self.in_, self.out, self.act, self.seq_len, self.height, self.width)


def param_shapes(L: Layer):
    """Shapes of the layer's parameter tensors, in flat-array order."""
    if L.kind == LINEAR:
        return [(L.out, L.in_), (L.out,)]
    if L.kind == LSTM:
        H = L.out
        return [(4 * H, L.in_), (4 * H, H), (4 * H,), (4 * H,)]
    if L.kind == CONV3X3:
        return [(L.out, L.in_, 3, 3), (L.out,)]
    if L.kind == EMBEDDING:
        return [(L.in_, L.out)]
    return []


def param_count(L: Layer) -> int:
    return int(sum(int(np.prod(s)) for s in param_shapes(L)))


@dataclass
class Workload:
    name: str
    layers: List[Layer]
    batch: int
    optimizer: int = SGD
    lr: float = 0.05
    beta1: float = 0.9
    beta2: float = 0.999
    eps: float = 1e-8
    # stage partition (index of each stage's last layer) and replication, when fixed
    stage_last: Optional[List[int]] = None
    replicas: Optional[List[int]] = None
    notes: str = ""
    extra: dict = field(default_factory=dict)

    @property
    def tokens_in(self) -> bool:
        return self.layers[0].kind == EMBEDDING

    @property
    def seq_len(self) -> int:
        return max(L.seq_len for L in self.layers)

    def rows(self) -> int:
        last = self.layers[-1]
        return self.batch * (last.seq_len if last.seq_len > 0 else 1)

    def classes(self) -> int:
        return self.layers[-1].out

    def input_elems(self) -> int:
        L0 = self.layers[0]
        if L0.kind == EMBEDDING:
            return L0.seq_len * self.batch
        if L0.kind in (CONV3X3, MAXPOOL2):
            return self.batch * L0.height * L0.width * L0.in_
        if L0.kind == LSTM:
            return L0.seq_len * self.batch * L0.in_
        return self.batch * (L0.seq_len if L0.seq_len else 1) * L0.in_


# ---------------------------------------------------------------------------
# BASELINE.json configs (full size) and their reduced parity versions
# ---------------------------------------------------------------------------

def mlp(widths, batch, relu_last=False):
    layers = []
    for i in range(len(widths) - 1):
        last = i == len(widths) - 2
        act = ACT_RELU if (not last or relu_last) else ACT_NONE
        layers.append(Layer(LINEAR, widths[i], widths[i + 1], act))
    return layers


def gnmt(n_lstm, hidden, vocab, seq, batch):
    layers = [Layer(EMBEDDING, vocab, hidden, seq_len=seq)]
    layers += [Layer(LSTM, hidden, hidden, seq_len=seq) for _ in range(n_lstm)]
    layers.append(Layer(LINEAR, hidden, vocab, ACT_NONE, seq_len=seq))
    return layers


def vgg(blocks, in_hw, in_c, fc, classes):
    """blocks: list of lists of conv output channels; a 2x2 max-pool follows each block."""
    layers, c, hw = [], in_c, in_hw
    for blk in blocks:
        for co in blk:
            layers.append(Layer(CONV3X3, c, co, ACT_RELU, height=hw, width=hw))
            c = co
        layers.append(Layer(MAXPOOL2, c, c, height=hw, width=hw))
        hw //= 2
    feat = hw * hw * c
    for f in fc:
        layers.append(Layer(LINEAR, feat, f, ACT_RELU))
        feat = f
    layers.append(Layer(LINEAR, feat, classes, ACT_NONE))
    return layers


VGG16_BLOCKS = [[64, 64], [128, 128], [256, 256, 256], [512, 512, 512], [512, 512, 512]]


def workload(name: str, reduced: bool = False) -> Workload:
    """The five BASELINE.json configs; ``reduced`` gives the parity-size variant."""
    if name == "mlp_small":  # cfg 1: 784-512-512-10 fp32, 2 stages, B=16, 8 minibatches
        return Workload(name, mlp([784, 512, 512, 10], 16), 16, SGD, 0.05,
                        stage_last=[1, 2], replicas=[1, 1])
    if name == "mlp4096":  # cfg 2: 16 x Linear(4096) bf16, B=256
        w = 64 if reduced else 4096
        b = 32 if reduced else 256
        return Workload(name, mlp([w] * 17, b), b, SGD, 0.5 if reduced else 0.01)
    if name in ("gnmt8", "gnmt16"):  # cfg 3 / 5: H=1024, T=50, V=32k, B=64, Adam 3e-4
        n = 8 if name == "gnmt8" else 16
        if reduced:
            return Workload(name, gnmt(n, 32, 64, 5, 4), 4, ADAM, 1e-2)
        return Workload(name, gnmt(n, 1024, 32000, 50, 64), 64, ADAM, 3e-4)
    if name == "vgg16":  # cfg 4: VGG-16 224^2 NHWC, B=64, SGD 0.01, 7-1
        if reduced:
            layers = vgg([[8], [16]], 8, 3, [32], 10)
            return Workload(name, layers, 4, SGD, 0.05)
        layers = vgg(VGG16_BLOCKS, 224, 3, [4096, 4096], 1000)
        return Workload(name, layers, 64, SGD, 0.01)
    raise KeyError(name)


# ---------------------------------------------------------------------------
# Seeded inputs and initial weights
# ---------------------------------------------------------------------------

def init_params(layers: List[Layer], seed: int = WEIGHT_SEED) -> List[np.ndarray]:
    """One flat fp32 array per layer, U(-1/sqrt(fan_in), 1/sqrt(fan_in))."""
    rng = np.random.default_rng(seed)
    out = []
    for L in layers:
        if L.kind == MAXPOOL2:
            out.append(np.zeros(0, np.float32))
            continue
        if L.kind == EMBEDDING:
            out.append(rng.standard_normal(param_count(L), dtype=np.float32))
            continue
        fan_in = {LINEAR: L.in_, LSTM: L.out, CONV3X3: L.in_ * 9}[L.kind]
        bound = 1.0 / np.sqrt(fan_in)
        out.append(rng.uniform(-bound, bound, param_count(L)).astype(np.float32))
    return out


def make_data(wl: Workload, n_data: int, seed: int = DATA_SEED):
    """n_data minibatches: (inputs fp32 or None, tokens int32 or None, labels int32)."""
    rng = np.random.default_rng(seed)
    inputs = tokens = None
    if wl.tokens_in:
        V = wl.layers[0].in_
        tokens = rng.integers(0, V, size=(n_data, wl.input_elems()), dtype=np.int32)
    else:
        inputs = rng.standard_normal((n_data, wl.input_elems()), dtype=np.float32)
    labels = rng.integers(0, wl.classes(), size=(n_data, wl.rows()), dtype=np.int32)
    return inputs, tokens, labels


def random_profile(rng: np.random.Generator, n_layers: int):
    """A random per-layer profile (T_l seconds, a_l bytes, w_l bytes) for planner tests."""
    T = rng.uniform(1e-4, 1e-2, n_layers)
    a = rng.integers(1 << 10, 1 << 26, n_layers).astype(np.uint64)
    w = rng.integers(0, 1 << 28, n_layers).astype(np.uint64)
    return T, a, w

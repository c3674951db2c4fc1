"""Parity at the bench's full sizes (VERDICT r1 "next round" #2): the 16-layer H = 1024
wavefront, the default long-K weight-gradient path (K = T*B = 3200) and the packed-tap VGG
conv1 at 224 x 224, each one bf16 SGD step of a single stage against the oracle's sampled
deltas (tests/golden/<case>.npz, written by tests/gen_golden_fullsize.py from oracle/ only).

Tolerances: parameters within the north star's bf16 2e-2 (max relative error); the deltas
(= -lr x gradient, where a version or indexing bug would show) within DELTA_TOL of the
floored delta norm (R23, "bf16 tolerance"), and the first loss within 1e-2.
DELTA_TOL: bf16 rounding alone (tools/bf16_emulate.py: torch fp64 with bf16 rounding where the
CUDA path stores bf16) puts the first layer's gradient of these random-label problems 5.4 %
(long-K W0) and 7.4 % (conv1 W) away from the exact one -- the gradient is a sum with heavy
cancellation -- and the GPU lands on those floors to 3 digits (measured: 0.0539 / 0.0739);
0.1 leaves room for accumulation order, not for a bug (a wrong version or index moves the
delta by O(1))."""
import os

import numpy as np
import pytest

import synth
import fullsize_cases as fc
import paper_conf_sosp_narayananhpsdgg19_b200 as pd
from paper_conf_sosp_narayananhpsdgg19_b200.session import Pipeline

pytestmark = pytest.mark.gpu

GOLDEN = os.path.join(os.path.dirname(os.path.abspath(__file__)), "golden")
DELTA_TOL = 0.1


@pytest.mark.parametrize("name", ["longk_dw", "vgg_conv1", "gnmt16_wave"])
def test_fullsize_one_step(name):
    g = np.load(os.path.join(GOLDEN, f"{name}.npz"))
    wl = fc.workload(name)
    p0 = synth.init_params(wl.layers)
    data = synth.make_data(wl, 1)
    with Pipeline(pd.Plan.manual([len(wl.layers) - 1], [1]), wl.layers, p0, dtype=pd.PD_BF16,
                  optimizer=wl.optimizer, lr=wl.lr, minibatch=wl.batch) as P:
        P.set_data(*data, 1)
        P.run(1)
        loss = float(P.losses(1)[0])
        got = P.params([synth.param_count(L) for L in wl.layers])
    errs = fc.sampled_errors(g, got)
    perr = max(float(np.abs(got[int(k.split("_")[0])][int(g[f"{k}_start"]) + g[f"{k}_pos"]] -
                            (g[f"{k}_p0"] + g[f"{k}_dref"])).max() / g[f"{k}_pmax"]) for k in g["keys"])
    worst = max(errs, key=errs.get)
    print(name, "loss", loss, float(g["loss"][0]), "param err", perr, "worst delta err", worst, errs[worst])
    assert abs(loss - float(g["loss"][0])) <= 1e-2 * abs(float(g["loss"][0])), (loss, float(g["loss"][0]))
    assert perr < 2e-2, perr
    assert errs[worst] < DELTA_TOL, errs

"""The sampled full-size goldens (tests/golden/<case>.npz) are the oracle's: for the cases the
single-threaded oracle finishes in seconds, recompute them here and require the stored
samples to match exactly (gnmt16_wave takes ~8 minutes and is only checked for structure)."""
import os

import numpy as np
import pytest

import oracle
import synth
import fullsize_cases as fc

GOLDEN = os.path.join(os.path.dirname(os.path.abspath(__file__)), "golden")


@pytest.mark.parametrize("name", ["longk_dw", "vgg_conv1"])
def test_golden_equals_a_fresh_oracle_run(name):
    g = np.load(os.path.join(GOLDEN, f"{name}.npz"))
    wl = fc.workload(name)
    p0 = synth.init_params(wl.layers)
    ref = oracle.run(wl.layers, [len(wl.layers) - 1], [1], wl.batch, 1, p0, synth.make_data(wl, 1), wl.optimizer,
                     wl.lr)
    assert float(g["loss"][0]) == float(ref.losses[0])
    for key in g["keys"]:
        l, k = (int(x) for x in str(key).split("_"))
        a = int(g[f"{key}_start"])
        pos = g[f"{key}_pos"]
        d = ref.params[l].astype(np.float64) - p0[l].astype(np.float64)
        assert np.array_equal(d[a + pos], g[f"{key}_dref"])


def test_gnmt16_golden_structure():
    g = np.load(os.path.join(GOLDEN, "gnmt16_wave.npz"))
    layers = fc.workload("gnmt16_wave").layers
    assert len(g["keys"]) == len(fc.tensor_slices(layers))  # every parameter tensor sampled
    assert np.isfinite(g["loss"]).all() and 5.0 < float(g["loss"][0]) < 7.0  # ~ln(512) at init

#!/usr/bin/env python
"""Writes tests/golden/<case>.npz: the oracle's one-step parameter deltas of a full-size case
(tests/fullsize_cases.py), sampled.  Calls only oracle/ and synth/ -- no value here comes
from the CUDA path.  The oracle is single-threaded; gnmt16_wave takes ~8 minutes.

    python tests/gen_golden_fullsize.py gnmt16_wave [more cases]
"""
import os
import sys
import time

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))  # repo root
sys.path.insert(0, ROOT)
sys.path.insert(0, os.path.dirname(os.path.abspath(__file__)))

import oracle  # noqa: E402
import synth  # noqa: E402
import fullsize_cases as fc  # noqa: E402


def main(name):
    wl = fc.workload(name)
    p0 = synth.init_params(wl.layers)
    data = synth.make_data(wl, 1)
    t0 = time.time()
    ref = oracle.run(wl.layers, [len(wl.layers) - 1], [1], wl.batch, 1, p0, data, wl.optimizer, wl.lr)
    dt = time.time() - t0
    out = {"keys": [], "loss": ref.losses[:1].astype(np.float64), "oracle_s": dt}
    keys = []
    for si, (l, k, a, b) in enumerate(fc.tensor_slices(wl.layers)):
        p_ref = ref.params[l][a:b].astype(np.float64)
        d_full = p_ref - p0[l][a:b].astype(np.float64)
        pos = fc.sample_positions(d_full, b - a, seed=1000 + si)
        key = f"{l}_{k}"
        keys.append(key)
        out[f"{key}_start"] = a
        out[f"{key}_pos"] = pos
        out[f"{key}_dref"] = d_full[pos]
        out[f"{key}_p0"] = p0[l][a:b][pos].astype(np.float64)
        out[f"{key}_dmax"] = np.abs(d_full).max()
        out[f"{key}_pmax"] = np.abs(p_ref).max()
    out["keys"] = np.array(keys)
    path = os.path.join(ROOT, "tests", "golden", f"{name}.npz")
    np.savez_compressed(path, **out)
    print(f"{name}: oracle {dt:.1f} s, loss {ref.losses[0]:.6f}, {len(keys)} tensors -> {path}")


if __name__ == "__main__":
    for n in sys.argv[1:]:
        main(n)

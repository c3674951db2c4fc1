#!/usr/bin/env python
"""Per-tensor view of how visible weight stashing is on the bf16 path (tests/stash_cases.py
design): for a case and a set of learning rates / minibatch counts, prints per parameter
tensor the delta error (R23) of
    gpu   : this library's bf16 run           vs the stashing oracle
    nost  : this library's bf16 run           vs the no-stash oracle
    mut   : the no-stash oracle               vs the stashing oracle
With PD_LIBRARY pointing at a fault-injected build it shows what the fault changes.
    python tools/stash_sweep.py mlp256 0.5,1.0 16,32 [bf16|fp32]
"""
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
sys.path.insert(0, os.path.join(ROOT, "tests"))

import numpy as np  # noqa: E402

import oracle  # noqa: E402
import synth  # noqa: E402
import stash_cases  # noqa: E402
import paper_conf_sosp_narayananhpsdgg19_b200 as pd  # noqa: E402
from gpu_helpers import run_both  # noqa: E402


def per_tensor(out, ref, init, floor=1e-2):
    errs = []
    for o, r, i in zip(out, ref, init):
        o, r, i = (np.asarray(x, np.float64) for x in (o, r, i))
        if r.size == 0:
            continue
        den = max(np.abs(r - i).max(), floor * np.abs(r).max(), 1e-30)
        errs.append(round(float(np.abs((o - i) - (r - i)).max() / den), 4))
    return errs


def main(name, lrs, Ms, dtype):
    wl0, last, reps, _M = stash_cases.case(name)
    for lr in lrs:
        for M in Ms:
            wl = synth.Workload(wl0.name, wl0.layers, wl0.batch, wl0.optimizer, lr)
            res = run_both(wl, last, reps, M, pd.PD_BF16 if dtype == "bf16" else pd.PD_FP32, n_data=4)
            p0, ref = res["p0"], res["ref"]
            mut = oracle.run(wl.layers, last, reps, wl.batch, M, p0, synth.make_data(wl, 4), wl.optimizer, lr,
                             stash=False)
            print(json.dumps({"case": name, "lr": lr, "M": M, "dtype": dtype,
                              "l2": {"gpu": stash_cases.rel_l2(res["got"], ref.params, p0),
                                     "nost": stash_cases.rel_l2(res["got"], mut.params, p0),
                                     "mut": stash_cases.rel_l2(mut.params, ref.params, p0)},
                              "gpu": per_tensor(res["got"], ref.params, p0),
                              "nost": per_tensor(res["got"], mut.params, p0),
                              "mut": per_tensor(mut.params, ref.params, p0)}), flush=True)


if __name__ == "__main__":
    main(sys.argv[1], [float(x) for x in sys.argv[2].split(",")], [int(x) for x in sys.argv[3].split(",")],
         sys.argv[4] if len(sys.argv) > 4 else "bf16")

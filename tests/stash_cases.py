"""bf16 pipelines in which weight stashing is VISIBLE ("what's weak" #1).

At the parity learning rates of the older bf16 tests the oracle's no-stash mutant stays
inside the 2e-2 tolerance, so those tests could not fail on a version bug.  The cases below
are chosen (on the CPU oracle, before any GPU run) so that reading the latest instead of
the stashed version moves the parameter deltas by far more than bf16
rounding does:

    case              no-stash mutant delta error (oracle vs oracle, R23)
    mlp256            0.21   4 x Linear(256)+ReLU, B 64, 4 single-layer stages, SGD 0.5
    mlp256_first1     -      same layers, stages [0 | 1..3]: single-layer first stage whose
                             overlapped backward has no dX to fork the side stream
    gnmt_adam         1.2    reduced GNMT-8 (Emb, 8 LSTM(32), Linear), 4 stages, Adam 1e-2
    vgg               0.33   reduced VGG (conv8+pool, conv16+pool, FC32, FC16), 2 stages, SGD 0.2
    vgg_31            0.19   same, conv stage replicated 3-1 (replica rounds), SGD 0.2

The criterion (test_gpu_stash_bf16.py): delta error of the GPU run against the stashing
oracle <= 1/4 of the mutant's, and > 1/4 of it against the no-stash oracle.

Run as a script (``python tests/stash_cases.py <case>``) it prints one JSON line of
errors; the negative-control tests run it with PD_LIBRARY pointing at a fault-injected
library (build.py FAULTS) and require the criterion to FAIL.
"""
from __future__ import annotations

import json
import os
import sys

HERE = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, HERE)
sys.path.insert(0, os.path.dirname(HERE))

import synth  # noqa: E402


def case(name):
    """(workload, stage_last, replicas, M)"""
    if name in ("mlp256", "mlp256_first1"):
        wl = synth.Workload(name, synth.mlp([256] * 5, 64), 64, synth.SGD, 0.5)
        return wl, ([0, 1, 2, 3] if name == "mlp256" else [0, 3]), ([1] * 4 if name == "mlp256" else [1, 1]), 16
    if name == "gnmt_adam":
        g = synth.workload("gnmt8", reduced=True)
        return synth.Workload(name, g.layers, g.batch, synth.ADAM, 1e-2), [2, 5, 8, 9], [1] * 4, 12
    if name in ("vgg", "vgg_31"):
        wl = synth.Workload(name, synth.vgg([[8], [16]], 8, 3, [32], 16), 4, synth.SGD, 0.2)
        return (wl, [2, 5], [1, 1], 9) if name == "vgg" else (wl, [3, 5], [3, 1], 12)
    raise KeyError(name)


CASES = ["mlp256", "mlp256_first1", "gnmt_adam", "vgg", "vgg_31"]


def evaluate(name):
    """Runs the case on the GPU (bf16) and both oracles; returns a dict of errors."""
    import oracle
    import torchref
    import paper_conf_sosp_narayananhpsdgg19_b200 as pd
    from gpu_helpers import run_both
    wl, last, reps, M = case(name)
    res = run_both(wl, last, reps, M, pd.PD_BF16, n_data=4)
    ref = res["ref"]
    p0 = res["p0"]
    data = synth.make_data(wl, 4)
    mut = oracle.run(wl.layers, last, reps, wl.batch, M, p0, data, wl.optimizer, wl.lr, wl.beta1, wl.beta2, wl.eps,
                     stash=False)
    got = [t[:8] for t in res["trace"]]
    return {
        "case": name,
        "trace_exact": got == ref.events,
        "param_err": torchref.max_rel_err(res["got"], ref.params),
        "delta_err": torchref.delta_err(res["got"], ref.params, p0),
        "delta_err_vs_nostash": torchref.delta_err(res["got"], mut.params, p0),
        "mutant_delta_err": torchref.delta_err(mut.params, ref.params, p0),
    }


def discriminates(r):
    """The bar: within 1/4 of the mutant's distance of the stashing oracle, and farther than
    that from the no-stash oracle."""
    q = r["mutant_delta_err"] / 4
    return r["delta_err"] <= q and r["delta_err_vs_nostash"] > q


if __name__ == "__main__":
    try:
        out = evaluate(sys.argv[1])
        out["discriminates"] = discriminates(out)
    except Exception as e:  # a fault-injected library may also fail loudly
        out = {"case": sys.argv[1], "error": f"{type(e).__name__}: {e}"}
    print(json.dumps(out), flush=True)

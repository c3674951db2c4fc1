"""Per-stage checkpointing: every worker dumps its own state with no
global coordination; restarting from the checkpoint continues training exactly where the
uninterrupted run goes (parameters, versions, optimizer step)."""
import os
import tempfile

import numpy as np
import pytest

import oracle
import synth
import torchref
import paper_conf_sosp_narayananhpsdgg19_b200 as pd
from paper_conf_sosp_narayananhpsdgg19_b200.session import Pipeline

pytestmark = pytest.mark.gpu

CASES = [
    ("mlp_small", [1, 2], [1, 1], 8, pd.PD_FP32, 0.0),        # deterministic SIMT path: bit-exact
    ("mlp256", [1, 3], [1, 1], 8, pd.PD_BF16, 0.0),           # tcgen05 + fused SGD, graphs
    ("gnmt8r", [2, 5, 8, 9], [1, 1, 1, 1], 8, pd.PD_BF16, 1e-5),  # Adam state; per-step fp32 atomics
    ("mlp4096r", [7, 15], [2, 1], 8, pd.PD_BF16, 0.0),        # replicated stage: sharded m, v
]


def _wl(name):
    if name == "mlp_small":
        return synth.workload("mlp_small")
    if name == "mlp256":
        return synth.Workload(name, synth.mlp([256] * 5, 64), 64, synth.SGD, 0.05)
    if name == "gnmt8r":
        return synth.workload("gnmt8", reduced=True)
    return synth.workload("mlp4096", reduced=True)


@pytest.mark.parametrize("name,last,reps,M,dtype,tol", CASES)
def test_checkpoint_restart_continues_training(name, last, reps, M, dtype, tol):
    wl = _wl(name)
    p0 = synth.init_params(wl.layers)
    data = synth.make_data(wl, 4)
    sizes = [synth.param_count(L) for L in wl.layers]
    plan = pd.Plan.manual(last, reps)
    kw = dict(dtype=dtype, optimizer=wl.optimizer, lr=wl.lr, minibatch=wl.batch)
    with tempfile.TemporaryDirectory() as d:
        with Pipeline(plan, wl.layers, p0, **kw) as P:
            P.set_data(*data, 4)
            P.run(M)
            P.save_checkpoint(d)
            assert len([f for f in os.listdir(d) if f.endswith(".pdckpt")]) == sum(reps)
            P.run(M)
            uninterrupted = P.params(sizes)
            vmap_a = P.version_map(M)
        junk = [np.zeros_like(p) for p in p0]  # the restarted run starts from different weights
        with Pipeline(plan, wl.layers, junk, **kw) as Q:
            Q.set_data(*data, 4)
            Q.load_checkpoint(d)
            Q.run(M)
            restarted = Q.params(sizes)
            vmap_b = Q.version_map(M)
    assert np.array_equal(vmap_a, vmap_b)  # versions continue from the checkpoint
    err = torchref.max_rel_err([restarted[l] for l in range(len(sizes))], [uninterrupted[l] for l in range(len(sizes))])
    assert err <= tol, err
    # and the two runs are the oracle's two consecutive runs
    r1 = oracle.run(wl.layers, last, reps, wl.batch, M, p0, data, wl.optimizer, wl.lr)
    if wl.optimizer == synth.SGD:  # (the oracle's Adam state restarts per run; SGD has none)
        r2 = oracle.run(wl.layers, last, reps, wl.batch, M, r1.params, data, wl.optimizer, wl.lr)
        tol2 = 1e-4 if dtype == pd.PD_FP32 else 2e-2
        assert torchref.max_rel_err([restarted[l] for l in range(len(sizes))], r2.params) < tol2


def test_load_checkpoint_rejects_a_mismatching_directory():
    wl = synth.workload("mlp_small")
    p0 = synth.init_params(wl.layers)
    with tempfile.TemporaryDirectory() as d:
        with Pipeline(pd.Plan.manual([1, 2], [1, 1]), wl.layers, p0, dtype=pd.PD_FP32, lr=wl.lr,
                      minibatch=wl.batch) as P:
            with pytest.raises(pd.PDError) as ei:
                P.load_checkpoint(d)  # no files
            assert ei.value.status == pd.PD_EINVAL

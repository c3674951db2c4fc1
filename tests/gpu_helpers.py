"""Shared helpers of the GPU parity tests: run a workload through the C ABI and through the
oracle on the same seeded inputs, and compare what the north star says must match."""
from __future__ import annotations

import numpy as np

import oracle
import synth
import torchref
import paper_conf_sosp_narayananhpsdgg19_b200 as pd
from paper_conf_sosp_narayananhpsdgg19_b200.session import Pipeline

FP32_TOL = 1e-4   # BASELINE.json north star, fp32 / tf32-off path
BF16_TOL = 2e-2   # bf16 path


def run_both(wl, stage_last, replicas, M, dtype, n_data=5, noam=0, lr=None, record_trace=1, device_of=None,
             sync_mode=0):
    lr = wl.lr if lr is None else lr
    p0 = synth.init_params(wl.layers)
    data = synth.make_data(wl, n_data)
    plan = pd.Plan.manual(stage_last, replicas)
    with Pipeline(plan, wl.layers, p0, dtype=dtype, optimizer=wl.optimizer, lr=lr, beta1=wl.beta1,
                  beta2=wl.beta2, eps=wl.eps, minibatch=wl.batch, record_trace=record_trace,
                  max_depth=noam, device_of=device_of, sync_mode=sync_mode) as P:
        P.set_data(*data, n_data)
        P.run(M, noam)
        sizes = [synth.param_count(L) for L in wl.layers]
        got = P.params(sizes)
        got = [got[l] for l in range(len(wl.layers))]
        trace = P.trace()
        vmap = P.version_map(M)
        losses = P.losses(M)
        stats = P.stats()
    ref = oracle.run(wl.layers, stage_last, replicas, wl.batch, M, p0, data, wl.optimizer, lr, wl.beta1,
                     wl.beta2, wl.eps, depth=noam, vertical_sync=sync_mode == pd.PD_SYNC_VERTICAL,
                     gpipe=sync_mode == pd.PD_SYNC_GPIPE)
    return dict(p0=p0, got=got, trace=trace, vmap=vmap, losses=losses, stats=stats, ref=ref)


def assert_schedule_exact(res):
    got = [t[:8] for t in res["trace"]]
    assert got == res["ref"].events, "event trace differs from the oracle"
    assert np.array_equal(res["vmap"], res["ref"].version_map), "version map differs from the oracle"


def param_errors(res):
    """(max relative error on params, floored relative error on deltas) -- DESIGN.md R23."""
    perr = torchref.max_rel_err(res["got"], res["ref"].params)
    derr = torchref.delta_err(res["got"], res["ref"].params, res["p0"])
    return perr, derr

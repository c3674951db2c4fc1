"""The B200 self-profiler (pd_profile, L841-847) and per-layer timing of pd_run, feeding the
partitioner."""
import numpy as np
import pytest

import synth
import paper_conf_sosp_narayananhpsdgg19_b200 as pd
from paper_conf_sosp_narayananhpsdgg19_b200.session import Pipeline

pytestmark = pytest.mark.gpu


def _mlp(width=1024, n=6, B=128):
    return synth.Workload("mlp", synth.mlp([width] * (n + 1), B), B, synth.SGD, 0.01)


def test_profile_fields_and_proportions():
    wl = _mlp()
    T, a, w = pd.pd_profile(wl.layers, pd.PD_BF16, wl.optimizer, wl.lr, wl.batch, 0, 6)
    assert len(T) == len(wl.layers)
    for l, L in enumerate(wl.layers):
        assert T[l] > 0
        assert a[l] == wl.batch * L.out * 2            # bf16 output activation (a_l)
        assert w[l] == 4 * synth.param_count(L)         # fp32 gradient bytes (w_l)
    inner = T[:-1]  # identical layers: similar times (the last one also carries the loss)
    assert max(inner) < 3 * min(inner), T
    # the profile describes the real single-stage run within a small factor (the real run
    # overlaps dW with dX and replays CUDA graphs; the profile serialises each layer)
    p0 = synth.init_params(wl.layers)
    data = synth.make_data(wl, 4)
    with Pipeline(pd.Plan.manual([len(wl.layers) - 1], [1]), wl.layers, p0, minibatch=wl.batch,
                  record_trace=2) as P:
        P.set_data(*data, 4)
        P.set_timing(2, 0)
        P.run(8)
        P.run(8)
        real = P.stats()["run_ms"] / 1e3 / 8
    assert 0.3 < real / sum(T) < 3.0, (real, sum(T))


def test_profile_feeds_the_partitioner():
    wl = _mlp(n=8)
    T, a, w = pd.pd_profile(wl.layers, pd.PD_BF16, wl.optimizer, wl.lr, wl.batch, 0, 4)
    for N in (2, 4):
        p = pd.pd_plan(T, a, w, N, max_replicas=1)
        assert [s[0] for s in p.stages][0] == 0 and p.stages[-1][1] == len(T) - 1
        assert len(p.stages) == N and p.noam == N
        # equal layers -> balanced straight partition
        sizes = [s[1] - s[0] + 1 for s in p.stages]
        assert max(sizes) - min(sizes) <= 1, sizes
        assert p.slowest_stage_s >= sum(T) / N * 0.999


def test_layer_times_on_a_pipeline():
    wl = synth.workload("gnmt8", reduced=True)
    p0 = synth.init_params(wl.layers)
    data = synth.make_data(wl, 4)
    with Pipeline(pd.Plan.manual([4, 9], [1, 1]), wl.layers, p0, dtype=pd.PD_BF16, optimizer=wl.optimizer,
                  lr=3e-4, minibatch=wl.batch) as P:
        P.set_data(*data, 4)
        P.set_layer_profiling(True)
        P.run(6)
        f, b = P.layer_times()
        P.set_layer_profiling(False)
        P.run(6)
    assert np.all(f > 0), f
    assert np.all(b[1:] > 0), b  # every layer has a backward (embedding: its dE scatter)

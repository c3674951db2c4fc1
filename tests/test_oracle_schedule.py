"""P3-P6 and the golden trace: the oracle's 1F1B-RR schedule against what PAPER.md fixes
(schedule-only mode, no math)."""
import os

import numpy as np
import pytest

import oracle
import synth
from synth import Layer, LINEAR

HERE = os.path.dirname(os.path.abspath(__file__))


def chain(n_layers):
    return [Layer(LINEAR, 4, 4)] * n_layers


def sched(stage_sizes, replicas, M, depth=0, fwd=None, bwd=None):
    layers = chain(sum(stage_sizes))
    last = list(np.cumsum(stage_sizes) - 1)
    return oracle.run(layers, last, replicas, 1, M, math=False, depth=depth, fwd_time=fwd, bwd_time=bwd)


def ops_of(res, stage, replica=0):
    return [f"{e[4]}{e[5]}" for e in res.events if e[1] == stage and e[2] == replica and e[4] != "U"]


# ---------------- P3: NOAM = ceil(workers / input-stage replicas) (L1021, L1045) ---------------

def test_noam_fig4_four_stages():
    assert oracle.inflight([1, 1, 1, 1])[0] == 4  # "The NOAM for this configuration is 4" L1045


def test_noam_fig8_two_one():
    assert oracle.inflight([2, 1])[0] == 2  # ceil(3/2), R1 (ceiling reading)


def test_noam_seven_one():
    assert oracle.inflight([7, 1])[0] == 2  # ceil(8/7)


def test_noam_pure_dp_and_model_parallel():
    assert oracle.inflight([8]) == [1]
    assert oracle.inflight([1, 1, 1, 1], depth=1) == [1, 1, 1, 1]


# ---------------- P4: event order (Fig. 4 / Fig. 8 / Fig. 9 text) ---------------

def test_fig4_input_stage_order():
    # startup admits exactly four minibatches, then B/F alternate (L1045-1065)
    r = sched([1, 1, 1, 1], [1, 1, 1, 1], 12)
    assert ops_of(r, 0)[:8] == ["F0", "F1", "F2", "F3", "B0", "F4", "B1", "F5"]
    assert ops_of(r, 1)[:6] == ["F0", "F1", "F2", "B0", "F3", "B1"]
    # the output stage runs its backward right after its forward (L1051-1055)
    assert ops_of(r, 3)[:6] == ["F0", "B0", "F1", "B1", "F2", "B2"]


def test_fig9_minibatch5_versions():
    # "minibatch 5 uses parameter updates from minibatch 1 on machine 1 and from 2 on
    # machine 2" (L1167-1169); 0-based t = 4, versions = number of updates applied.
    r = sched([1, 1, 1, 1], [1, 1, 1, 1], 12)
    assert list(r.version_map[:, 4]) == [1, 2, 3, 4]
    # L1121-1127 (no stashing): F of minibatch 5 on stage 1 follows the update of
    # minibatch 1; its backward comes after the updates of minibatches 2, 3, 4.
    ev0 = [e for e in r.events if e[1] == 0]
    order = [(e[4], e[5]) for e in ev0]
    f5, b5 = order.index(("F", 4)), order.index(("B", 4))
    ups_before_b5 = [e[5] for e in ev0[:b5] if e[4] == "U"]
    ups_before_f5 = [e[5] for e in ev0[:f5] if e[4] == "U"]
    assert ups_before_f5 == [0]
    assert ups_before_b5 == [0, 1, 2, 3]
    # ... but with weight stashing the backward reads the forward's version
    b = [e for e in ev0 if e[4] == "B" and e[5] == 4][0]
    assert b[6] == 1


def test_fig8_round_robin():
    # 2-1: even IDs to worker 1 (replica 0), odd to worker 2; worker 3 takes all (L1089-1097)
    r = sched([1, 1], [2, 1], 8)
    assert all(int(o[1:]) % 2 == 0 for o in ops_of(r, 0, 0))
    assert all(int(o[1:]) % 2 == 1 for o in ops_of(r, 0, 1))
    assert sorted(int(o[1:]) for o in ops_of(r, 1) if o[0] == "F") == list(range(8))
    # F and B of a minibatch run on the same replica (L1073-1077)
    for rep in (0, 1):
        fs = {o[1:] for o in ops_of(r, 0, rep) if o[0] == "F"}
        bs = {o[1:] for o in ops_of(r, 0, rep) if o[0] == "B"}
        assert fs == bs


def test_golden_cfg1_trace():
    gold = []
    with open(os.path.join(HERE, "golden", "cfg1_trace.txt")) as f:
        for line in f:
            if line.startswith("#") or not line.strip():
                continue
            s, k, t, vi, vo = line.split()
            gold.append((int(s), k, int(t), int(vi), int(vo)))
    wl = synth.workload("mlp_small")
    r = oracle.run(wl.layers, wl.stage_last, wl.replicas, wl.batch, 8, math=False)
    got = [(e[1], e[4], e[5], e[6], e[7]) for e in r.events]
    assert got == gold


# ---------------- P6: version map closed form ---------------

@pytest.mark.parametrize("stages,reps", [([1, 1], [1, 1]), ([1, 1, 1, 1], [1] * 4), ([2] * 8, [1] * 8),
                                         ([1, 1], [2, 1]), ([1, 1], [7, 1]), ([1, 1], [3, 1]), ([1], [4])])
def test_version_map_closed_form(stages, reps):
    M = 4 * int(np.lcm.reduce(reps)) * 6
    r = sched(stages, reps, M)
    k = oracle.inflight(reps)
    for s in range(len(stages)):
        for t in range(M):
            assert r.version_map[s, t] == max(0, t // reps[s] - k[s] + 1)


def test_version_map_equals_paper_superscripts():
    # straight pipeline: stage i (1-based) uses w_i^(t-n+i) (L1237-1241), clamped at 0 (R5)
    n, M = 5, 40
    r = sched([1] * n, [1] * n, M)
    for i in range(1, n + 1):
        for t in range(M):
            assert r.version_map[i - 1, t] == max(0, t - n + i)


# ---------------- P5: timelines (Fig. 2 / Fig. 4, footnote 4) ---------------

@pytest.mark.parametrize("F,B,n,M", [(1.0, 2.0, 4, 40), (2.0, 3.0, 4, 60), (1.0, 1.0, 3, 17), (1.0, 2.0, 8, 30)])
def test_balanced_makespan_and_bubble_closed_form(F, B, n, M):
    r = sched([1] * n, [1] * n, M, fwd=[F] * n, bwd=[B] * n)
    assert r.makespan == pytest.approx((M + n - 1) * (F + B), abs=1e-9)
    assert r.bubble == pytest.approx((n - 1) / (M + n - 1), abs=1e-12)


def _steady_idle(r, n, k0):
    idle = 0.0
    for s in range(n):
        ts = [tuple(x) for e, x in zip(r.events, r.times) if e[1] == s and e[4] != "U"]
        ts = ts[k0:-k0]
        idle += sum(max(0.0, b[0] - a[1]) for a, b in zip(ts, ts[1:]))
    return idle


@pytest.mark.parametrize("F,B", [(1.0, 2.0), (2.0, 3.0)])
def test_steady_state_has_no_idle(F, B):
    # "every worker is performing either a forward or backward pass" (L1061-1065); also for
    # a non-integer backward:forward ratio such as 3:2 (footnote 4, L1149)
    n, M = 4, 40
    r = sched([1] * n, [1] * n, M, fwd=[F] * n, bwd=[B] * n)
    assert _steady_idle(r, n, 2 * n) == 0.0


def test_model_parallel_one_worker_busy():
    # Fig. 2: without pipelining at most one worker is active (L375-381, L491-519)
    n, M = 4, 6
    r = sched([1] * n, [1] * n, M, depth=1, fwd=[1.0] * n, bwd=[2.0] * n)
    iv = [tuple(x) for e, x in zip(r.events, r.times) if e[4] != "U"]
    for a in iv:
        for b in iv:
            if a is not b and a != b:
                assert a[1] <= b[0] or b[1] <= a[0]
    assert r.bubble == pytest.approx(0.75)


def test_replicated_input_stage_balanced_no_idle():
    # 2-1 from Fig. 8: stage 0 takes two time units per pass, stage 1 one (L949-955)
    r = sched([1, 1], [2, 1], 40, fwd=[2.0, 1.0], bwd=[2.0, 1.0])
    n_busy = sum(e - s for s, e in r.times)
    assert r.bubble < 0.1 and n_busy > 0


def test_schedule_counts():
    for stages, reps in [([1, 1, 1, 1], [1] * 4), ([1, 1], [7, 1])]:
        M = 28
        r = sched(stages, reps, M)
        for s in range(len(stages)):
            for kind in "FBU":
                cnt = sum(1 for e in r.events if e[1] == s and e[4] == kind)
                assert cnt == M

"""P8: the oracle's §3.1 partitioner (L899-985) against brute-force enumeration written
independently here, plus closed-form special cases."""
import itertools
import time

import numpy as np
import pytest

import oracle
import synth

BW = 900e9


def stage_time(T, w, i, j, m, bw, comm_model):
    # T(i->j, m) per DESIGN.md R11 (literal: comm not divided by m inside the max)
    comp = sum(T[i:j + 1])
    ws = float(sum(int(x) for x in w[i:j + 1]))
    comm = 2 * (m - 1) * ws / (m * bw) if comm_model == 1 else 2 * (m - 1) * ws / bw
    return max(comp, comm) / m


def objective(T, a, w, bounds, reps, bw, comm_model):
    """slowest stage of a whole plan = max over stages and stage boundaries (R10, R12)."""
    vals = []
    first = 0
    for q, (last, m) in enumerate(zip(bounds, reps)):
        vals.append(stage_time(T, w, first, last, m, bw, comm_model))
        if q + 1 < len(bounds):
            vals.append(2.0 * float(a[last]) / bw)
        first = last + 1
    return max(vals)


def brute_force(T, a, w, gpus, bw=BW, max_rep=0, comm_model=0):
    N = len(T)
    maxr = max_rep or gpus
    best, arg = None, []
    for n in range(1, N + 1):
        for cuts in itertools.combinations(range(N - 1), n - 1):
            bounds = list(cuts) + [N - 1]
            for reps in itertools.product(range(1, maxr + 1), repeat=n):
                if sum(reps) != gpus:
                    continue
                v = objective(T, a, w, bounds, reps, bw, comm_model)
                if best is None or v < best * (1 - 1e-12):
                    best, arg = v, [(bounds, list(reps))]
                elif v <= best * (1 + 1e-12):
                    arg.append((bounds, list(reps)))
    return best, arg


@pytest.mark.parametrize("seed", range(60))
def test_dp_equals_brute_force(seed):
    rng = np.random.default_rng(seed)
    N = int(rng.integers(1, 7))
    gpus = int(rng.integers(1, 5))
    T, a, w = synth.random_profile(rng, N)
    bw = float(rng.choice([1e9, 25e9, 900e9]))
    for max_rep in (0, 1):
        for cm in (0, 1):
            best, arg = brute_force(T, a, w, gpus, bw, max_rep, cm)
            if best is None:  # e.g. straight pipeline with fewer layers than GPUs
                with pytest.raises(ValueError):
                    oracle.plan(T, a, w, gpus, bw, max_rep, cm)
                continue
            p = oracle.plan(T, a, w, gpus, bw, max_rep, cm)
            assert p.slowest == pytest.approx(best, rel=1e-12)
            assert (p.stage_last, p.replicas) in [(b, r) for b, r in arg]
            assert sum(p.replicas) == gpus
            assert p.noam == -(-gpus // p.replicas[0])


def test_zero_comm_free_choice_is_pure_dp():
    # with no weight/activation bytes, a single stage replicated m ways gives sum(T)/m
    T = np.array([3e-3, 1e-3, 2e-3, 5e-3])
    z = np.zeros(4, np.uint64)
    p = oracle.plan(T, z, z, 4, BW)
    assert p.stage_last == [3] and p.replicas == [4]
    assert p.slowest == pytest.approx(T.sum() / 4, rel=1e-15)
    assert p.noam == 1


def test_straight_zero_comm_is_minmax_linear_partition():
    rng = np.random.default_rng(7)
    T = rng.uniform(1, 10, 9)
    z = np.zeros(9, np.uint64)
    for k in (2, 3, 4):
        p = oracle.plan(T, z, z, k, BW, max_replicas=1)
        best = min(max(sum(T[i:j]) for i, j in zip((0,) + c, c + (9,)))
                   for c in itertools.combinations(range(1, 9), k - 1))
        assert p.slowest == pytest.approx(best, rel=1e-12)
        assert p.replicas == [1] * k and p.noam == k


def test_heavy_weights_avoid_replication():
    # a layer with a huge weight and tiny activations should not be replicated (cf. L737-747)
    T = np.array([1e-3, 1e-3, 1e-3, 1e-3])
    a = np.array([1 << 20] * 4, np.uint64)
    w = np.array([1 << 20, 1 << 20, 1 << 20, 1 << 34], np.uint64)
    p = oracle.plan(T, a, w, 4, 25e9)
    assert p.replicas[-1] == 1


def test_infeasible_raises():
    with pytest.raises(ValueError):
        oracle.plan([1.0, 1.0], [0, 0], [0, 0], 3, BW, max_replicas=1)


def test_runtime_under_8s_for_40_layers_8_gpus():
    # "the running time is under 8 seconds" (L985)
    rng = np.random.default_rng(0)
    T, a, w = synth.random_profile(rng, 40)
    t0 = time.time()
    oracle.plan(T, a, w, 8, BW)
    assert time.time() - t0 < 8.0

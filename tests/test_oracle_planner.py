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


# ---------------------------------------------------------------- hierarchical topology (Fig. 7)

def hier_brute(T, a, w, levels, max_rep=0, comm_model=0):
    """A^L(0 -> N-1, m_L) by exhaustive enumeration at every level (no optimal-substructure
    shortcut): a level-k plan is any contiguous partition with replication factors summing
    to m_k; a stage's compute is the best level-(k-1) plan of its layers on a whole level-(k-1)
    component (level 0: the sum of T_l) -- L865-899, L903-975 as read in DESIGN.md R10-R16."""
    import functools
    N = len(T)

    @functools.lru_cache(maxsize=None)
    def A(k, i, j):
        if k < 0:
            return sum(T[i:j + 1])
        mk, bw = levels[k]
        maxr = max_rep or mk
        best = None
        n_l = j - i + 1
        for n in range(1, n_l + 1):
            for cuts in itertools.combinations(range(i, j), n - 1):
                bounds = list(cuts) + [j]
                for reps in itertools.product(range(1, min(maxr, mk) + 1), repeat=n):
                    if sum(reps) != mk:
                        continue
                    vals, first = [], i
                    for q, (last, m) in enumerate(zip(bounds, reps)):
                        ws = float(sum(int(x) for x in w[first:last + 1]))
                        comm = 2 * (m - 1) * ws / (m * bw) if comm_model == 1 else 2 * (m - 1) * ws / bw
                        vals.append(max(A(k - 1, first, last), comm) / m)
                        if q + 1 < len(bounds):
                            vals.append(2.0 * float(a[last]) / bw)
                        first = last + 1
                    v = max(vals)
                    if best is None or v < best:
                        best = v
        return best if best is not None else float("inf")

    return A(len(levels) - 1, 0, N - 1)


@pytest.mark.parametrize("seed", range(24))
def test_hierarchical_dp_equals_brute_force(seed):
    rng = np.random.default_rng(100 + seed)
    N = int(rng.integers(1, 6))
    T, a, w = synth.random_profile(rng, N)
    levels = [[(2, 900e9), (2, 25e9)], [(3, 900e9), (2, 12.5e9)], [(2, 600e9), (2, 50e9), (2, 10e9)]][seed % 3]
    for max_rep in (0, 1):
        bf = hier_brute(T, a, w, levels, max_rep)
        if bf == float("inf"):
            with pytest.raises(ValueError):
                oracle.plan_levels(T, a, w, levels, max_replicas=max_rep)
            continue
        p = oracle.plan_levels(T, a, w, levels, max_replicas=max_rep)
        assert p.slowest == pytest.approx(bf, rel=1e-12, abs=0)
        gpus = int(np.prod([m for m, _ in levels]))
        assert sum(p.replicas) == gpus and p.stage_last[-1] == N - 1
        assert p.noam == -(-gpus // p.replicas[0])
        if max_rep == 1:
            assert all(r == 1 for r in p.replicas)


@pytest.mark.parametrize("seed", range(12))
def test_one_level_hierarchy_is_the_flat_dp(seed):
    """levels = [(G, B)] is the single-level partitioner exactly (m_0 = 1, A^0 = sum T_l)."""
    rng = np.random.default_rng(200 + seed)
    N, G = int(rng.integers(1, 7)), int(rng.integers(1, 6))
    T, a, w = synth.random_profile(rng, N)
    for mr in (0, 1):
        try:
            flat = oracle.plan(T, a, w, G, 25e9, max_replicas=mr)
        except ValueError:
            with pytest.raises(ValueError):
                oracle.plan_levels(T, a, w, [(G, 25e9)], max_replicas=mr)
            continue
        lev = oracle.plan_levels(T, a, w, [(G, 25e9)], max_replicas=mr)
        assert (lev.stage_last, lev.replicas, lev.noam, lev.slowest) == (flat.stage_last, flat.replicas, flat.noam,
                                                                          flat.slowest)


def test_hierarchical_infeasible_component_stays_infeasible():
    """A range that has no plan on one level-(k-1) component (one layer, 4 GPUs, at most 2
    replicas per stage) has none on several of them either: replicating an infeasible
    component plan m' times must not look finite (the max / m of R10-R11 with an infinite
    compute term)."""
    T, a, w = [1e-3], [1 << 20], [1 << 20]
    assert hier_brute(T, a, w, [(4, 900e9), (2, 25e9)], max_rep=2) == float("inf")
    with pytest.raises(ValueError):
        oracle.plan_levels(T, a, w, [(4, 900e9), (2, 25e9)], max_replicas=2)

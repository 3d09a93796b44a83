"""NEXT #1 — round-based scheduler (CPU): the C++ implementation against the plain oracle
(oracle/sched.py) and the oracle's DP against exhaustive search (App. B)."""
import itertools
import math

import numpy as np
import pytest

from oracle import sched as OS

KS = [1, 2, 4, 8]


def random_table(rng, n_res=4):
    # T(res, k) shaped like a DiT step: sublinear scaling in k (Insight 2)
    base = np.array([0.02, 0.05, 0.2, 1.0])[:n_res] * rng.uniform(0.8, 1.2, n_res)
    eff = np.array([1.0, 0.9, 0.75, 0.55]) * rng.uniform(0.9, 1.0, 4)
    T = base[:, None] / (np.array(KS)[None, :] * eff[None, :])
    return T


@pytest.fixture(scope="module")
def sched():
    import __graft_entry__
    __graft_entry__.build()
    from paper_conf_asplos_luhtlwm0c26_b200 import sched as S
    return S


def test_allocate_matches_oracle(sched):
    rng = np.random.default_rng(0)
    for _ in range(200):
        T = random_table(rng)
        row = int(rng.integers(0, 4))
        steps = int(rng.integers(1, 21))
        N = int(rng.choice([1, 2, 4, 8]))
        budget = float(rng.uniform(0.2, 1.2)) * steps * T[row, 0]
        spk, late = sched.allocate(T, KS, budget, steps, row, 0.0, N)
        ref = OS.allocate(T[row], KS, steps, budget, N)
        if ref is None:
            assert late
            assert sum(spk) == steps
        else:
            assert not late
            got = sorted((s, k) for s, k in zip(spk, KS) if s)
            assert got == sorted(ref)


def test_allocation_optimality_brute_force():
    """The oracle's allocation is the exact optimum of eq. (checked on small S against an
    independent enumeration over per-step degree sequences)."""
    rng = np.random.default_rng(1)
    for _ in range(50):
        T = random_table(rng)[0]
        steps = int(rng.integers(1, 6))
        budget = float(rng.uniform(0.3, 1.1)) * steps * T[0]
        best = None
        for seq in itertools.product(range(4), repeat=steps):
            time = sum(T[j] for j in seq)
            if time <= budget + 1e-12:
                cost = sum(KS[j] * T[j] for j in seq)
                best = cost if best is None else min(best, cost)
        ref = OS.allocate(T, KS, steps, budget, 8)
        if best is None:
            assert ref is None
        else:
            assert math.isclose(sum(s * k * T[KS.index(k)] for s, k in ref), best, rel_tol=1e-9)


def _instance(rng, R, N):
    T = random_table(rng)
    reqs = []
    for _ in range(R):
        row = int(rng.integers(0, 4))
        steps = int(rng.integers(1, 21))
        deadline = float(rng.uniform(0.1, 1.5)) * steps * T[row, 0]
        reqs.append((deadline, steps, row))
    return T, reqs


def test_dp_equals_exhaustive():
    """Alg. 1's group-knapsack DP attains the optimum of the per-round problem (exhaustive search,
    App. B) on small instances (R <= 6, N <= 8)."""
    rng = np.random.default_rng(2)
    for _ in range(300):
        R, N = int(rng.integers(1, 7)), int(rng.choice([1, 2, 4, 8]))
        T, raw = _instance(rng, R, N)
        tau = float(rng.uniform(0.05, 0.5))
        reqs = []
        for d, s, row in raw:
            t_of = {k: t for k, t in zip(KS, T[row]) if k <= N}
            alloc = OS.allocate(T[row], KS, s, d, N) or [(s, 1)]
            reqs.append(dict(alloc=alloc, T=lambda A, t_of=t_of: t_of[A], T_min=min(t_of.values()), deadline=d))
        v, plan = OS.dp_round(reqs, tau, 0.0, N)
        assert v == OS.exhaustive_round(reqs, tau, 0.0, N)
        assert sum(w for _, _, w in plan) <= N


def test_round_matches_oracle(sched):
    rng = np.random.default_rng(3)
    for _ in range(300):
        R, N = int(rng.integers(0, 9)), int(rng.choice([1, 2, 4, 8]))
        T, reqs = _instance(rng, R, N)
        tau = float(rng.uniform(0.05, 0.5))
        now = float(rng.uniform(0, 0.05))
        for wc in (False, True):
            got = sched.schedule_round(T, KS, reqs, now, tau, N, work_conserving=wc)
            ref = OS.schedule_round(T, KS, reqs, now, tau, N, work_conserving=wc)
            assert got[0] == ref[0]
            assert got[1] == [tuple(x) for x in ref[1]]
            assert sum(g for g, _ in got[1]) <= N


def test_round_work_conserving_tie(sched):
    """Alg. 1 line 21 tie: a request with ample slack survives with or without running, so the
    smallest-capacity optimum (S31) defers it while the largest-capacity one (S31b) runs it now at
    its minimal allocation; the survivor count is the same."""
    T = np.array([[1.0, 0.6, 0.35, 0.2]])
    reqs = [(100.0, 5, 0)]
    sv0, plan0 = sched.schedule_round(T, KS, reqs, 0.0, 1.0, 8)
    sv1, plan1 = sched.schedule_round(T, KS, reqs, 0.0, 1.0, 8, work_conserving=True)
    assert sv0 == sv1 == 1
    assert plan0 == [(0, 0)] and plan1 == [(1, 1)]


def test_round_semantics(sched):
    T = np.array([[1.0, 0.6, 0.35, 0.2]])
    # a single request that can only meet its deadline at k = 8 gets 8 GPUs
    sv, plan = sched.schedule_round(T, KS, [(0.2 * 5 + 1e-9, 5, 0)], 0.0, 1.0, 8)
    assert plan == [(8, 5)] and sv == 1
    # with only 4 GPUs it is late: best effort on one GPU
    sv, plan = sched.schedule_round(T, KS, [(1.0, 5, 0)], 0.0, 1.0, 4)
    assert plan == [(1, 1)] and sv == 0
    # bad arguments
    with pytest.raises(Exception):
        sched.schedule_round(T, KS, [(1.0, 5, 3)], 0.0, 1.0, 4)


def test_scheduler_latency(sched):
    """Decision time stays far below the paper's < 10 ms for 64 requests on 8 GPUs."""
    import time
    rng = np.random.default_rng(4)
    T, reqs = _instance(rng, 64, 8)
    t0 = time.perf_counter()
    for _ in range(10):
        sched.schedule_round(T, KS, reqs, 0.0, 0.25, 8)
    assert (time.perf_counter() - t0) / 10 < 0.010


# ----------------------------------------------------------------------------- placement (NEXT #4)
def _rand_plan(rng, N):
    sizes = []
    left = N
    while left > 0 and rng.random() < 0.8:
        g = int(rng.choice([k for k in KS if k <= left]))
        sizes.append(g)
        left -= g
    sizes += [0] * int(rng.integers(0, 3))
    rng.shuffle(sizes)
    return sizes


def test_place_matches_oracle(sched):
    rng = np.random.default_rng(5)
    for _ in range(500):
        N = int(rng.choice([2, 4, 8, 16]))
        T = random_table(rng)
        gpus = _rand_plan(rng, N)
        R = len(gpus)
        rows = [int(rng.integers(0, 4)) for _ in range(R)]
        prev = [set(int(x) for x in rng.choice(N, size=int(rng.integers(0, N + 1)), replace=False)) for _ in range(R)]
        for up in (False, True):
            got = sched.place(T, KS, rows, gpus, prev, N, up)
            ref = OS.place(T, KS, rows, gpus, prev, N, up)
            assert got == ref
            used = set()
            for i, b in enumerate(got):
                assert not (b & used)                       # disjoint
                used |= b
                if b:
                    g, s = len(b), min(b)
                    assert b == set(range(s, s + g)) and s % g == 0   # aligned power-of-two block
                    assert g >= gpus[i] if up else g == gpus[i]
                else:
                    assert gpus[i] == 0
            if up:   # work-conserving: GPUs stay idle only if every request already has some
                assert len(used) == N or all(got)


def test_place_preserves_previous_blocks(sched):
    T = np.array([[1.0, 0.6, 0.35, 0.2]])
    # same sizes as last round and those blocks are free: every request keeps its GPUs
    prev = [{4, 5, 6, 7}, {2, 3}, {1}]
    got = sched.place(T, KS, [0, 0, 0], [4, 2, 1], prev, 8, False)
    assert got == prev
    # elastic scale-up: the idle GPU 0 doubles the 1-GPU request in place (buddy of {1})
    got = sched.place(T, KS, [0, 0, 0], [4, 2, 1], prev, 8, True)
    assert got == [{4, 5, 6, 7}, {2, 3}, {0, 1}]
    # no gain from a larger degree: no scale-up
    Tflat = np.array([[1.0, 1.0, 1.0, 1.0]])
    assert sched.place(Tflat, KS, [0], [1], [set()], 8, True) == [{0}]
    with pytest.raises(Exception):
        sched.place(T, KS, [0, 0], [8, 1], [set(), set()], 8, False)   # over capacity

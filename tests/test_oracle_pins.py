"""Pins for the oracle (CPU, -m "not gpu").

Each test checks the oracle against something other than itself: values
printed in the paper, hand derivations, closed forms, invariants that the
mathematics fixes, or brute force on tiny inputs (exhaustive m^n assignment,
exhaustive set-partition bin packing).  None restates the oracle's own loop.
"""
from __future__ import annotations

import itertools
import json
import math
import os

import numpy as np
import pytest

import oracle
from synth import jobs

GOLD = os.path.join(os.path.dirname(__file__), "golden")


def _gold(name):
    with open(os.path.join(GOLD, name)) as f:
        return json.load(f)


# ---------------------------------------------------------------- k, bounds
def test_k_values():
    # PAPER.md:68 k = ceil(1/eps); eps=0.3 -> k=4 gives "k^2 = 16 dims"
    assert oracle.k_of(0.3) == 4
    assert oracle.k_of(0.2) == 5
    assert oracle.k_of(0.15) == 7
    assert oracle.k_of(0.25) == 4
    assert oracle.k_of(0.1) == 10
    assert oracle.k_of(0.5) == 2
    assert oracle.k_of(1.0) == 1


def test_bounds_hand():
    # Alg 1 l.2-3: sum=10, m=2 -> ceil=5, max=5
    assert oracle.bounds([3, 5, 2], 2) == (5, 10)
    # sum=7, m=3 -> ceil(7/3)=3, max=4 -> LB=4, UB=7
    assert oracle.bounds([4, 2, 1], 3) == (4, 7)
    # single job: LB = p, UB = 2p
    assert oracle.bounds([9], 5) == (9, 11)


# ---------------------------------------------------------------- classify
def test_classify_hand():
    # T=100, k=4: u = floor(100/16) = 6; 26 is long (104 > 100) -> 24;
    # 25 is short (100 is not > 100) (reading i-1); 100 -> 96 (16*6)
    u, r, N, cls = oracle.classify([26, 25, 100, 27], 100, 4)
    assert u == 6
    assert list(r) == [24, 96]
    assert list(N) == [2, 1]
    assert list(cls) == [0, -1, 1, 0]
    # T < k^2: u = max(1, floor(T/k^2)) = 1 (reading i-2), rounding exact
    u, r, N, cls = oracle.classify([3, 2, 5], 10, 4)
    assert u == 1
    assert list(r) == [3, 5]
    assert list(cls) == [0, -1, 1]


def test_classify_no_long_jobs():
    u, r, N, cls = oracle.classify([1, 2, 3], 1000, 4)
    assert len(r) == 0 and (cls == -1).all()


# ---------------------------------------------------------------- configs
def test_configs_uncapacitated_counts_paper_example():
    # "(1,2,1) has eleven sub-configurations, and (0,0,4) has only four"
    # -> candidates are all s <= v except s = 0 (reading i-4).
    assert len(oracle.configs([1, 2, 1], [1, 1, 1], 10**9)) == 11
    assert len(oracle.configs([0, 0, 4], [1, 1, 1], 10**9)) == 4


@pytest.mark.parametrize("N,r,T", [(7, 30, 100), (2, 30, 100), (5, 101, 1000), (0, 5, 5)])
def test_configs_K1_closed_form(N, r, T):
    assert len(oracle.configs([N], [r], T)) == min(N, T // r)


def test_configs_bruteforce_full_box():
    rng = np.random.default_rng(1)
    for _ in range(60):
        K = int(rng.integers(1, 5))
        N = rng.integers(0, 5, K)
        r = rng.integers(1, 40, K)
        T = int(rng.integers(int(r.max()), 120))
        got = [tuple(x) for x in oracle.configs(N, r, T)]
        want = [s for s in itertools.product(*[range(int(x) + 1) for x in N])
                if any(s) and sum(a * b for a, b in zip(s, r)) <= T]
        assert got == want  # same set, lexicographic order


def test_configs_bounded_size_when_u_gt_k():
    # every s in C has |s| <= k when u > k (T >= k^2 (k+1)): long jobs have r > T/k - u ... survey §8c-ii
    for seed in range(20):
        p = jobs(40, 1000, seed)
        k = 4
        T = 2000
        u, r, N, cls = oracle.classify(p, T, k)
        assert u > k
        C = oracle.configs(N, r, T)
        assert (C.sum(axis=1) <= k).all()


# ---------------------------------------------------------------- DP table
def test_g1_table_hand():
    g = _gold("g1_table.json")
    tab, relax = oracle.dp(g["N"], g["r"], g["T"])
    assert tab.tolist() == g["table"]
    assert relax == g["relax"]
    assert oracle.configs(g["N"], g["r"], g["T"]).tolist() == g["configs_lex"]


def _min_bins_all_subsets(items, T):
    """Exhaustive set partition of distinguishable items into bins of capacity T:
    best[mask] = min #bins.  Bins are enumerated as submasks containing the
    lowest item of the mask (every partition is reached)."""
    n = len(items)
    load = [0] * (1 << n)
    for mask in range(1, 1 << n):
        low = mask & -mask
        load[mask] = load[mask ^ low] + items[low.bit_length() - 1]
    INF = 10**9
    best = [INF] * (1 << n)
    best[0] = 0
    for mask in range(1, 1 << n):
        low = mask & -mask
        rest = mask ^ low
        sub = rest
        while True:
            b = sub | low
            if load[b] <= T and best[mask ^ b] + 1 < best[mask]:
                best[mask] = best[mask ^ b] + 1
            if sub == 0:
                break
            sub = (sub - 1) & rest
    return best


def test_dp_equals_exhaustive_bin_packing_every_entry():
    # OPT(n) = min number of bins of capacity T packing {n_i x r_i} (PAPER.md:79:
    # "minimum number of machines sufficient to schedule the set of jobs ... within T")
    rng = np.random.default_rng(7)
    checked = 0
    for _ in range(60):
        K = int(rng.integers(1, 5))
        N = rng.integers(0, 4, K)
        while N.sum() > 10 or N.sum() == 0:
            N = rng.integers(0, 4, K)
        r = rng.integers(5, 60, K)
        T = int(rng.integers(int(r.max()), 150))
        tab, _ = oracle.dp(N, r, T)
        items = []
        first = []
        for i in range(K):
            first.append(len(items))
            items += [int(r[i])] * int(N[i])
        best = _min_bins_all_subsets(items, T)
        for n in itertools.product(*[range(int(x) + 1) for x in N]):
            mask = 0
            for i in range(K):
                for t in range(n[i]):
                    mask |= 1 << (first[i] + t)
            assert tab[n] == best[mask], (N, r, T, n)
            checked += 1
    assert checked > 500


@pytest.mark.parametrize("N,r,T", [(17, 30, 100), (40, 7, 50), (9, 100, 100), (0, 3, 3), (255, 11, 100)])
def test_dp_K1_closed_form(N, r, T):
    tab, _ = oracle.dp([N], [r], T)
    per = T // r
    assert [int(v) for v in tab] == [math.ceil(x / per) for x in range(N + 1)]


def _random_small(rng):
    K = int(rng.integers(1, 5))
    N = rng.integers(0, 6, K)
    r = rng.integers(10, 70, K)
    T = int(rng.integers(int(r.max()), 200))
    return N, r, T


def test_dp_invariants():
    rng = np.random.default_rng(11)
    for _ in range(40):
        N, r, T = _random_small(rng)
        tab, _ = oracle.dp(N, r, T)
        K = len(N)
        assert tab[(0,) * K] == 0
        for n in itertools.product(*[range(int(x) + 1) for x in N]):
            v = int(tab[n])
            # lower bound: total rounded load / T
            assert v >= math.ceil(sum(a * b for a, b in zip(n, r)) / T)
            for i in range(K):
                if n[i] < N[i]:
                    m_ = list(n)
                    m_[i] += 1
                    w = int(tab[tuple(m_)])
                    assert v <= w <= v + 1          # monotone, +1 Lipschitz
                e = [0] * K
                e[i] = 1
                if N[i] >= 1:
                    assert tab[tuple(e)] == 1        # r_i <= T
        # subadditivity on all a + b <= N
        pts = list(itertools.product(*[range(int(x) + 1) for x in N]))
        for a in pts[:: max(1, len(pts) // 25)]:
            for b in pts:
                s = tuple(x + y for x, y in zip(a, b))
                if all(s[i] <= N[i] for i in range(K)):
                    assert tab[s] <= tab[a] + tab[b]


def test_relaxation_closed_form():
    # relax = sum_{s in C} prod_i (N_i - s_i + 1): each s is
    # dominated by exactly prod (N_i - s_i + 1) table entries.
    rng = np.random.default_rng(3)
    for _ in range(40):
        N, r, T = _random_small(rng)
        _, relax = oracle.dp(N, r, T)
        C = oracle.configs(N, r, T)
        closed = sum(int(np.prod(N - s + 1)) for s in C)
        assert relax == closed


def test_dp_row_major_equals_brute_recursion():
    # plain memoised recursion of Eq. 1 from the top (a different evaluation order)
    import functools
    rng = np.random.default_rng(5)
    for _ in range(20):
        N, r, T = _random_small(rng)
        C = [tuple(int(x) for x in s) for s in oracle.configs(N, r, T)]
        tab, _ = oracle.dp(N, r, T)

        @functools.lru_cache(None)
        def opt(n):
            if not any(n):
                return 0
            return 1 + min(opt(tuple(a - b for a, b in zip(n, s)))
                           for s in C if all(b <= a for a, b in zip(n, s)))
        for n in itertools.product(*[range(int(x) + 1) for x in N]):
            assert tab[n] == opt(n)


# ---------------------------------------------------------------- search + schedule
def _brute_cmax(p, m):
    """Exact optimum makespan by enumerating all m^n assignments (vectorised)."""
    n = len(p)
    idx = np.arange(m ** n)
    loads = np.zeros((m ** n, m), np.int64)
    for j in range(n):
        d = (idx // (m ** j)) % m
        loads[np.arange(m ** n), d] += p[j]
    return int(loads.max(axis=1).min())


def _pred(p, m, k, T):
    u, r, N, cls = oracle.classify(p, T, k)
    if len(N) == 0:
        return True, 0
    tab, _ = oracle.dp(N, r, T)
    opt = int(tab[tuple(N)])
    return opt <= m, opt


def _check_schedule(p, m, eps, res):
    k = oracle.k_of(eps)
    Ts = res["T_star"]
    a = res["assignment"]
    assert len(a) == len(p) and (a >= 0).all() and (a < m).all()
    loads = np.bincount(a, weights=p, minlength=m)
    assert int(loads.max()) == res["makespan"]
    u, r, N, cls = oracle.classify(p, Ts, k)
    long_load = np.zeros(m, np.int64)
    for j in range(len(p)):
        if cls[j] >= 0:
            long_load[a[j]] += r[cls[j]]
    assert long_load.max() <= Ts  # each machine's rounded long load fits T*


def test_ptas_bruteforce_guarantee_and_search_invariants():
    # H-S guarantee makespan <= (1+eps) C*max ([16]) and
    # search invariants: pred(T*) holds; T* = LB0 or pred(T*-1) fails; T* <= C*max
    checked = 0
    for seed in range(60):
        p = jobs(10, 100, seed)
        m = 3
        eps = 0.3
        cmax = _brute_cmax(p, m)
        LB0, UB0 = oracle.bounds(p, m)
        k = oracle.k_of(eps)
        for P in (1, 2, 4):
            res = oracle.ptas(p, m, eps, P)
            Ts = res["T_star"]
            assert LB0 <= Ts <= UB0
            assert _pred(p, m, k, Ts)[0]
            if Ts > LB0:
                assert not _pred(p, m, k, Ts - 1)[0]
            assert Ts <= cmax
            assert res["makespan"] <= (1 + eps) * cmax + 1e-9
            _check_schedule(p, m, eps, res)
            checked += 1
    assert checked == 180


def test_alg1_bisection_sequence_P1():
    # P = 1 reproduces Alg 1: T = floor((LB+UB)/2); feasible -> UB = T else LB = T+1
    for seed in range(30):
        p = jobs(12, 100, seed)
        m, eps = 3, 0.3
        k = oracle.k_of(eps)
        LB, UB = oracle.bounds(p, m)
        seq = []
        while LB < UB:
            T = (LB + UB) // 2
            f, opt = _pred(p, m, k, T)
            seq.append((T, int(f), opt))
            if f:
                UB = T
            else:
                LB = T + 1
        res = oracle.ptas(p, m, eps, 1)
        assert [(t, f, o) for (t, _, f, _, o, _) in res["probes"]] == seq
        assert res["T_star"] == LB


def test_multisection_interval_shrinks():
    # Alg 3: "the size of the new interval is a quarter or even one-eighth"
    for seed in range(30):
        p = jobs(12, 100, seed)
        m = 3
        LB, UB = oracle.bounds(p, m)
        for P in (2, 4, 8):
            res = oracle.ptas(p, m, 0.3, P)
            rounds = {}
            for (T, rd, f, *_rest) in res["probes"]:
                rounds.setdefault(rd, []).append((T, f))
            lb, ub = LB, UB
            for rd in sorted(rounds):
                pr = rounds[rd]
                assert len(pr) <= P
                assert all(lb <= T < ub for T, _ in pr)
                width = ub - lb
                feas = [T for T, f in pr if f]
                if feas:
                    nub = min(feas)
                    nlb = max([lb] + [T + 1 for T, f in pr if not f and T < nub])
                else:
                    nlb, nub = max(T for T, _ in pr) + 1, ub
                assert nub - nlb <= -(-width // P) + 1
                lb, ub = nlb, nub
            assert lb == ub == res["T_star"]


def test_golden_g2():
    g = _gold("g2_m1_seed0.json")
    assert oracle.bounds(g["p"], g["m"]) == (g["LB"], g["UB"])
    res = oracle.ptas(g["p"], g["m"], g["eps"], 1)
    assert [[T, f, o] for (T, _, f, _, o, _) in res["probes"]] == g["P1_probes"]
    assert res["T_star"] == g["T_star"] and res["makespan"] == g["makespan"]
    assert res["assignment"].tolist() == g["assignment"]
    u, r, N, _ = oracle.classify(g["p"], g["T_star"], g["k"])
    assert u == g["u"] and r.tolist() == g["r"] and N.tolist() == g["N"]
    res4 = oracle.ptas(g["p"], g["m"], g["eps"], 4)
    rounds = {}
    for (T, rd, *_r) in res4["probes"]:
        rounds.setdefault(rd, []).append(T)
    assert [rounds[i] for i in sorted(rounds)] == g["P4_rounds"]
    assert res4["T_star"] == g["T_star"] and res4["assignment"].tolist() == g["assignment"]
    assert _brute_cmax(np.array(g["p"]), g["m"]) == g["brute_force_Cmax"]


def test_golden_g3_nonmonotone():
    g = _gold("g3_nonmonotone.json")
    p = np.array(g["p"])
    k = g["k"]
    # the predicate flips back at T=71 -> 72 (reading i-9)
    assert _pred(p, g["m"], k, 71)[0] and not _pred(p, g["m"], k, 72)[0]
    q = g["nonmonotone_points"]["k4_m2"]
    assert _pred(np.array(q["p"]), 2, 4, q["T"][0])[0] != _pred(np.array(q["p"]), 2, 4, q["T"][1])[0]
    q = g["nonmonotone_points"]["k5_m3"]
    assert _pred(np.array(q["p"]), 3, 5, q["T"][0])[0] != _pred(np.array(q["p"]), 3, 5, q["T"][1])[0]
    for P, want in g["by_P"].items():
        res = oracle.ptas(p, g["m"], g["eps"], int(P))
        assert res["T_star"] == want["T_star"]
        assert res["makespan"] == want["makespan"]
        assert [[T, f] for (T, _, f, *_r) in res["probes"]] == want["probes"]
        assert res["makespan"] <= 1.4 * g["brute_force_Cmax"]
    assert _brute_cmax(p, g["m"]) == g["brute_force_Cmax"]


def test_empty_dp_path_literal_configs():
    # BASELINE.json configs 2-5 literal: no long job at T = LB
    from synth import WORKLOADS
    for name in ("M2", "M3"):
        w = WORKLOADS[name]
        p = w.p()
        res = oracle.ptas(p, w.m, w.eps, 1)
        assert all(K == 0 for (_, _, _, K, _, _) in res["probes"])
        # with no long jobs the schedule is the greedy list schedule: makespan <= A + max p
        LB, UB = oracle.bounds(p, w.m)
        assert res["makespan"] <= UB


# ---------------------------------------------------------------- high-multiplicity bin packing
def test_hmbp_bins_equal_exhaustive_and_packing_valid():
    """oracle.hmbp: the bin count equals the exhaustive
    set-partition optimum, and the packing is a valid partition: every bin
    holds at most T, no bin is empty, per-class totals equal N."""
    rng = np.random.default_rng(71)
    for _ in range(50):
        K = int(rng.integers(1, 5))
        N = rng.integers(0, 4, K)
        while N.sum() > 10 or N.sum() == 0:
            N = rng.integers(0, 4, K)
        r = rng.integers(5, 60, K)
        T = int(rng.integers(int(r.max()), 150))
        bins, pk = oracle.hmbp(N, r, T)
        items = [int(r[i]) for i in range(K) for _ in range(int(N[i]))]
        assert bins == _min_bins_all_subsets(items, T)[(1 << len(items)) - 1]
        assert pk.shape == (bins, K)
        assert (pk.sum(axis=0) == N).all()
        assert ((pk * r).sum(axis=1) <= T).all() and (pk.sum(axis=1) > 0).all()


def test_hmbp_closed_forms_and_edges():
    # K = 1: ceil(N / floor(T / r)) bins; reading R11 takes the smallest s that
    # keeps OPT(n - s) = OPT(n) - 1 first (2 of 17, then full bins of 3)
    bins, pk = oracle.hmbp([17], [30], 100)
    assert bins == 6 and pk[:, 0].tolist() == [2, 3, 3, 3, 3, 3]
    # zero counts and an all-zero instance
    assert oracle.hmbp([0, 0], [5, 7], 10)[0] == 0
    bins, pk = oracle.hmbp([0, 4], [50, 5], 10)
    assert bins == 2 and (pk[:, 0] == 0).all()
    # load bound ceil(32 / 10) = 4 is met: {6,4} {6,4} {3,3,3} {3}
    bins, _ = oracle.hmbp([2, 2, 4], [6, 4, 3], 10)
    assert bins == 4
    # 3 items of 5 and 3 of 4, capacity 9: every bin holds at most one 5 => 3 bins
    assert oracle.hmbp([3, 3], [5, 4], 9)[0] == 3
    with pytest.raises(ValueError):
        oracle.hmbp([1], [11], 10)   # an item larger than the capacity


# --- Alg 2 comparator (oracle/ptas_oracle_omp.c, bench.py's all-core cpu_baseline) ---

def test_dp_omp_equals_exhaustive_bin_packing():
    # pinned directly to bin packing, not only to oracle_dp
    rng = np.random.default_rng(17)
    for _ in range(30):
        K = int(rng.integers(1, 5))
        N = rng.integers(0, 4, K)
        while N.sum() > 10 or N.sum() == 0:
            N = rng.integers(0, 4, K)
        r = rng.integers(5, 60, K)
        T = int(rng.integers(int(r.max()), 150))
        tab, _ = oracle.dp_omp(N, r, T)
        items, first = [], []
        for i in range(K):
            first.append(len(items))
            items += [int(r[i])] * int(N[i])
        best = _min_bins_all_subsets(items, T)
        for n in itertools.product(*[range(int(x) + 1) for x in N]):
            mask = 0
            for i in range(K):
                for t in range(n[i]):
                    mask |= 1 << (first[i] + t)
            assert tab[n] == best[mask], (N, r, T, n)


@pytest.mark.parametrize("N,r,T", [(17, 30, 100), (255, 11, 100), (0, 3, 3)])
def test_dp_omp_K1_closed_form(N, r, T):
    tab, _ = oracle.dp_omp([N], [r], T)
    per = T // r
    assert [int(v) for v in tab] == [math.ceil(x / per) for x in range(N + 1)]


def test_dp_omp_equals_oracle_dp_and_relax_closed_form():
    rng = np.random.default_rng(23)
    for _ in range(12):
        K = int(rng.integers(2, 7))
        N = rng.integers(1, 9, K)
        r = rng.integers(20, 120, K)
        T = int(rng.integers(int(r.max()) * 2, 500))
        a, ra = oracle.dp(N, r, T)
        b, rb = oracle.dp_omp(N, r, T)
        assert np.array_equal(a, b)
        C = oracle.configs(N, r, T)
        assert ra == rb == sum(int(np.prod(N - s + 1)) for s in C)
    assert oracle.omp_threads() >= 1

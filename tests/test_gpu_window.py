"""Level window (D15): OPT(N) of
Eq. 1 with only min(N0, T/r0) + 1 slabs of the first internal class resident
(a ring mapped twice in virtual memory).  Every value is compared with the
oracle: OPT(N) of random tables, the golden OPT of the M4x / M3g tables under a
budget below their full size, and whole solves whose probe DPs all run
windowed (the schedule's DP at T* is a full table)."""
from __future__ import annotations

import json
import os

import numpy as np
import pytest

import oracle
from synth import WORKLOADS, jobs

pytestmark = pytest.mark.gpu
GOLD = os.path.join(os.path.dirname(__file__), "golden", "shaped")


@pytest.fixture(scope="module")
def P():
    import paper_conf_ipps_ligsg18_b200 as P
    return P


def test_window_opt_random_vs_oracle(P):
    rng = np.random.default_rng(2024)
    used = 0
    for it in range(80):
        K = int(rng.integers(2, 7))
        N = rng.integers(1, {2: 60, 3: 25, 4: 12, 5: 8, 6: 6}[K], K).astype(np.int32)
        if it % 7 == 0:
            N[rng.integers(0, K)] += 250            # uint16 tables
        r = rng.integers(20, 200, K).astype(np.int64)
        T = int(rng.integers(int(r.max()), int(r.max()) * 4))
        opt, st = P.dp_fill_opt(N, r, T, window=1)
        tab, _ = oracle.dp(N, r, T)
        assert opt == int(tab[tuple(N)]), (N.tolist(), r.tolist(), T)
        used += st["window_dps"]
        full, st2 = P.dp_fill_opt(N, r, T, window=-1)
        assert full == opt and st2["window_dps"] == 0
        # (memory: the window's slabs are rounded up to the 2 MB mapping granularity,
        # so tiny tables use more; the saving is checked on the large tables below)
    assert used > 40


@pytest.mark.parametrize("name,budget", [("M4x", 1 << 30), ("M3g", 3 << 30)])
def test_window_table_beyond_budget(P, name, budget):
    """The full table (M4x 1.75 GB, M3g 5.5 GB) exceeds the budget; the windowed
    DP fits it and returns the oracle's OPT(N) (tests/golden/shaped)."""
    g = json.load(open(os.path.join(GOLD, f"table_{name}.json")))
    N, r, T = np.asarray(g["N"], np.int32), np.asarray(g["r"], np.int64), g["T"]
    assert g["sigma"] * g["e"] > budget
    with pytest.raises(P.PtasError) as ei:
        P.dp_fill_opt(N, r, T, budget=budget, window=-1)
    assert ei.value.rc == -2
    opt, st = P.dp_fill_opt(N, r, T, budget=budget, window=0)
    assert opt == g["opt"] and st["window_dps"] == 1 and 0 < st["dev_bytes_max"] <= budget
    assert st["relaxations"] == g["relax"]


@pytest.mark.parametrize("name", ["M2s", "M5s-0.3"])
def test_window_solve_vs_oracle_golden(P, name):
    w = WORKLOADS[name]
    g = json.load(open(os.path.join(GOLD, f"solve_{name}_P1.json")))
    got = P.ptas_solve(w.p(), w.m, w.eps, P=1, window=1)
    assert got["T_star"] == g["T_star"] and got["makespan"] == g["makespan"]
    assert got["assignment"].tolist() == g["assignment"]
    assert [list(x[:6]) for x in got["probes"]] == g["probes"]
    assert got["stats"]["window_dps"] > 0


def test_window_solve_small_vs_oracle(P):
    for seed in range(10):
        p = jobs(40, 1000, seed)
        got = P.ptas_solve(p, 8, 0.3, P=2, window=1)
        want = oracle.ptas(p, 8, 0.3, 2)
        assert got["T_star"] == want["T_star"] and got["assignment"].tolist() == want["assignment"].tolist()


def test_window_tstar_must_fit(P):
    # probes beyond the budget run windowed, but the schedule needs DP(T*) in full
    w = WORKLOADS["M2s"]
    with pytest.raises(P.PtasError) as ei:
        P.ptas_solve(w.p(), w.m, w.eps, P=1, budget=40 << 20)
    assert ei.value.rc == -2

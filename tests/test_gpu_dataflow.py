"""GPU parity of the dataflow fill (D7): one launch per run of
row-levels, row sets from a ticket counter, per-row ready flags.

Same bit-exact comparisons against the oracle as test_gpu_parity.py, with
PTAS_DF = 1 (the whole DP in one launch), PTAS_DF = 2 (runs of small
row-levels between per-level launches; a tiny PTAS_DF_ROWS splits every DP
into several runs), PTAS_DF = 3 (block row sets for narrow levels) and
PTAS_DF = 4 (narrow levels by one thread-block cluster in lockstep).
"""
from __future__ import annotations

import numpy as np
import pytest

import oracle
from synth import WORKLOADS, jobs
from test_gpu_parity import _check_table, _cmp_solve, _rand_case, _subbox

pytestmark = pytest.mark.gpu

# (PTAS_DF, PTAS_DF_ROWS, PTAS_DF_SPLIT_ROWS)
MODES = [("1", None, None), ("2", "40", None), ("2", "3000", None),
         ("3", None, None), ("3", None, "20"), ("3", None, "1000000000"),
         ("4", None, None), ("4", None, "1000000000"), ("4c2", None, "1000000000")]


@pytest.fixture(scope="module")
def P():
    import paper_conf_ipps_ligsg18_b200 as P
    return P


@pytest.fixture(params=MODES, ids=lambda m: f"df{m[0]}-rows{m[1]}-split{m[2]}")
def df(request, monkeypatch):
    mode, rows, split = request.param
    if mode == "4c2":   # cluster runs with a 2-CTA cluster: many sets per warp and level
        mode = "4"
        monkeypatch.setenv("PTAS_CL_SIZE", "2")
    monkeypatch.setenv("PTAS_DF", mode)
    if rows is not None:
        monkeypatch.setenv("PTAS_DF_ROWS", rows)
    if split is not None:
        monkeypatch.setenv("PTAS_DF_SPLIT_ROWS", split)
    return request.param


@pytest.mark.parametrize("K", [2, 3, 4, 5, 6, 7, 8, 9])
def test_df_random_uint8(P, df, K):
    rng = np.random.default_rng(3000 + K)
    maxN = {2: 60, 3: 25, 4: 12, 5: 8, 6: 6, 7: 4, 8: 3, 9: 3}[K]
    for _ in range(8):
        N, r, T = _rand_case(rng, K, maxN)
        _check_table(P, N, r, T)


@pytest.mark.parametrize("K", [2, 3, 4])
def test_df_random_uint16(P, df, K):
    rng = np.random.default_rng(4000 + K)
    for _ in range(3):
        N = rng.integers(1, {2: 200, 3: 60, 4: 20}[K], K).astype(np.int32)
        N[-1] = max(int(N[-1]), 256 - int(N[:-1].sum()) + 1)
        r = rng.integers(20, 200, K).astype(np.int64)
        T = int(rng.integers(int(r.max()), int(r.max()) * 5))
        _check_table(P, N, r, T)


def test_df_shapes(P, df):
    # long rows, ragged chunks, long in-row chains, many tiny rows (deep level chains)
    _check_table(P, np.array([5, 4, 70], np.int32), np.array([90, 70, 11], np.int64), 200)
    _check_table(P, np.array([2, 120], np.int32), np.array([40, 3], np.int64), 150)
    _check_table(P, np.array([6, 5, 32], np.int32), np.array([40, 50, 30], np.int64), 160)
    _check_table(P, np.array([30, 40, 300], np.int32), np.array([90, 70, 11], np.int64), 200)
    _check_table(P, np.array([300, 200, 2], np.int32), np.array([60, 50, 40], np.int64), 170)
    _check_table(P, np.array([0, 3, 0, 4], np.int32), np.array([10, 20, 30, 40], np.int64), 60)
    for W in (1, 2, 3, 5, 9, 33, 65):
        _check_table(P, np.array([40, 30, W - 1], np.int32), np.array([35, 50, 21], np.int64), 110)


@pytest.mark.parametrize("ch", ["1", "2", "4"])
def test_df_lane_layouts(P, df, monkeypatch, ch):
    monkeypatch.setenv("PTAS_DF_CH", ch)
    for W in (3, 7, 20, 33, 61):
        _check_table(P, np.array([9, 8, W - 1], np.int32), np.array([35, 50, 21], np.int64), 110)


def test_df_two_word_packing(P, df, monkeypatch):
    monkeypatch.setenv("PTAS_FORCE_TWO_WORDS", "1")
    rng = np.random.default_rng(78)
    for K in (3, 5, 8):
        for _ in range(3):
            N, r, T = _rand_case(rng, K, {3: 20, 5: 6, 8: 3}[K])
            _check_table(P, N, r, T)


def test_df_solves(P, df):
    for seed in range(30):
        _cmp_solve(P, jobs(12, 100, seed), 3, 0.3, 1)
    for (n, m, eps, seed) in [(40, 8, 0.3, 1), (60, 14, 0.3, 2), (50, 10, 0.2, 3)]:
        for Pp in (1, 3):   # P > 1: concurrent DP slots, each with its own flags and ticket
            _cmp_solve(P, jobs(n, 1000, seed), m, eps, Pp)


@pytest.mark.parametrize("name", ["M2s", "M3s", "M5s-0.3"])
def test_df_full_size_sampled(P, df, name):
    """Full-size DP at T = LB in the bench's configuration: sub-box parity,
    sampled Eq. 1 checks, invariants on the whole table."""
    w = WORKLOADS[name]
    p = w.p()
    k = oracle.k_of(w.eps)
    LB, _ = oracle.bounds(p, w.m)
    u, r, N, _ = oracle.classify(p, LB, k)
    opt, tab, st = P.dp_fill(N, r, LB)
    t64 = tab.astype(np.int64)
    Nc = _subbox(N)
    want, _ = oracle.dp(Nc, r, LB)
    assert (t64[tuple(slice(0, int(x) + 1) for x in Nc)] == want).all()
    C = oracle.configs(N, r, LB)
    rng = np.random.default_rng(1)
    for _ in range(2000):
        n = np.array([rng.integers(0, x + 1) for x in N])
        if not n.any():
            continue
        cand = [t64[tuple(n - s)] for s in C if (s <= n).all()]
        assert t64[tuple(n)] == 1 + min(cand)
    assert t64.flat[0] == 0
    for ax in range(len(N)):
        d = np.diff(t64, axis=ax)
        assert d.min() >= 0 and d.max() <= 1
    assert opt == t64[tuple(N)]


def test_df_matches_level_launches_on_solve(P, monkeypatch):
    """Whole M2s solve: DF modes give the same probe log / schedule as per-level launches."""
    w = WORKLOADS["M2s"]
    monkeypatch.setenv("PTAS_DF", "0")
    ref = P.ptas_solve(w.p(), w.m, w.eps, P=1)
    for mode in ("1", "2", "3", "4"):
        monkeypatch.setenv("PTAS_DF", mode)
        got = P.ptas_solve(w.p(), w.m, w.eps, P=1)
        assert got["T_star"] == ref["T_star"] and got["makespan"] == ref["makespan"]
        assert (got["assignment"] == ref["assignment"]).all()
        assert [x[:5] for x in got["probes"]] == [x[:5] for x in ref["probes"]]
        assert got["stats"]["fill_launches"] < ref["stats"]["fill_launches"]

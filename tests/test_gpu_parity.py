"""GPU parity: the CUDA path (through the C ABI) against the oracle, bit-exact.

All tables are integer (uint8/uint16); comparisons are exact.  Sizes span
several warp chunks and ragged tails (rows longer than 32 with W % 32 != 0,
many rows per row-level, more rows than one wave of the grid).
"""
from __future__ import annotations

import itertools
import json
import os

import numpy as np
import pytest

import oracle
from synth import WORKLOADS, jobs

pytestmark = pytest.mark.gpu
GOLD = os.path.join(os.path.dirname(__file__), "golden")


@pytest.fixture(scope="module")
def P():
    import paper_conf_ipps_ligsg18_b200 as P
    return P


def _rand_case(rng, K, maxN, e16=False):
    N = rng.integers(0, maxN + 1, K).astype(np.int32)
    if e16:
        N[rng.integers(0, K)] += 256
    r = rng.integers(20, 200, K).astype(np.int64)
    T = int(rng.integers(int(r.max()), int(r.max()) * 6))
    return N, r, T


# ------------------------------------------------------------------ a-3
def test_configs_match_oracle(P):
    rng = np.random.default_rng(100)
    for trial in range(120):
        K = int(rng.integers(1, 10))
        N, r, T = _rand_case(rng, K, 6)
        got = P.dp_configs(N, r, T)
        want = oracle.configs(N, r, T)
        assert got.shape == want.shape and (got == want).all(), (N, r, T)


def test_configs_large_box(P):
    # many configurations (capacity admits ~k items of small classes)
    N = np.array([40, 30, 25, 20, 18, 15], np.int32)
    r = np.array([30, 37, 41, 53, 60, 71], np.int64)
    got = P.dp_configs(N, r, 400)
    want = oracle.configs(N, r, 400)
    assert len(want) > 1000 and (got == want).all()


# ------------------------------------------------------------------ a-4
def test_row_index_complete(P):
    rng = np.random.default_rng(5)
    for trial in range(30):
        K = int(rng.integers(1, 7))
        N = rng.integers(0, 9, K).astype(np.int32)
        ls, rb = P.dp_row_index(N)
        nz = N[N > 0]
        if len(nz) == 0:
            assert list(ls) == [0, 1] and list(rb) == [0]
            continue
        W = int(nz[-1]) + 1
        sigma = int(np.prod(nz.astype(np.int64) + 1))
        # level sizes = coefficients of prod_{i<K-1} (1 + z + ... + z^{N_i})
        poly = np.array([1], np.int64)
        for x in nz[:-1]:
            poly = np.convolve(poly, np.ones(int(x) + 1, np.int64))
        assert list(np.diff(ls)) == list(poly)
        # every row exactly once, in lexicographic order within a level
        assert sorted(rb.tolist()) == list(range(0, sigma, W))
        shape = tuple(int(x) + 1 for x in nz[:-1])
        for L in range(len(poly)):
            rows = rb[ls[L]:ls[L + 1]] // W
            digs = [np.unravel_index(int(q), shape) if shape else () for q in rows]
            assert all(sum(d) == L for d in digs)
            assert digs == sorted(digs)


# ------------------------------------------------------------------ a-5
def _collapsed_relax(N, r, T):
    """Closed form of the (n, s') window gathers the packed kernel evaluates
    (D5, D12, D13): one window per (row p, x) for every prefix s' != 0
    with s' <= p whose first nonzero digit q is also the first nonzero digit of
    p, i.e. prod_{i >= q} (N_i - s'_i + 1) rows; no in-row term; row 0 is a
    closed form.  Internal order = the non-empty classes."""
    nz = np.asarray(N) > 0
    Nn, rn = np.asarray(N)[nz].astype(np.int64), np.asarray(r)[nz]
    if len(Nn) == 0:
        return 0.0
    W = float(Nn[-1] + 1)
    C = oracle.configs(Nn.astype(np.int32), rn, T)
    pre = {tuple(int(x) for x in c[:-1]) for c in C} - {tuple([0] * (len(Nn) - 1))}
    tot = 0.0
    for s in pre:
        s = np.array(s, np.int64)
        q = int(np.argmax(s > 0))
        tot += float(np.prod((Nn[q:-1] - s[q:] + 1).astype(np.float64))) * W
    return tot


def _check_table(P, N, r, T):
    opt, tab, st = P.dp_fill(N, r, T)
    want, relax = oracle.dp(N, r, T)
    assert tab.shape == want.shape
    bad = np.argwhere(tab.astype(np.int64) != want)
    assert len(bad) == 0, (N.tolist(), r.tolist(), T, bad[:5].tolist())
    assert opt == int(want[tuple(N)]) if len(N) else opt == 0
    assert st["relaxations"] == relax
    # executed relaxations: the collapsed count on the packed kernel, the full one on the scalar kernel
    assert st["relax_executed"] in (relax, _collapsed_relax(N, r, T)), (st["relax_executed"], relax)
    nz = np.asarray(N)[np.asarray(N) > 0]
    if os.environ.get("PTAS_FORCE_SCALAR") == "1":
        assert st["relax_executed"] == relax
    elif len(nz) and (int(nz[-1]) + 1) * (1 if nz.sum() <= 255 else 2) <= 124:
        assert st["relax_executed"] == _collapsed_relax(N, r, T)   # packed kernel for sure
    return tab


def test_g1_golden(P):
    g = json.load(open(os.path.join(GOLD, "g1_table.json")))
    opt, tab, st = P.dp_fill(g["N"], g["r"], g["T"])
    assert tab.tolist() == g["table"]
    assert st["relaxations"] == g["relax"]
    assert opt == 2


@pytest.fixture(params=["default", "0"], ids=["df-default", "level-launches"])
def fillmode(request, monkeypatch):
    """default: the library's fill schedule (dataflow runs, D7);
    "0": one launch per row-level."""
    if request.param != "default":
        monkeypatch.setenv("PTAS_DF", request.param)
    return request.param


@pytest.mark.parametrize("K", [1, 2, 3, 4, 5, 6, 7, 8, 9])
def test_dp_fill_random_uint8(P, K, fillmode):
    rng = np.random.default_rng(1000 + K)
    maxN = {1: 200, 2: 60, 3: 25, 4: 12, 5: 8, 6: 6, 7: 4, 8: 3, 9: 3}[K]
    for _ in range(12):
        N, r, T = _rand_case(rng, K, maxN)
        _check_table(P, N, r, T)


@pytest.mark.parametrize("K", [1, 2, 3, 4])
def test_dp_fill_random_uint16(P, K, fillmode):
    rng = np.random.default_rng(2000 + K)
    for _ in range(4):
        N = rng.integers(1, {1: 300, 2: 200, 3: 60, 4: 20}[K], K).astype(np.int32)
        N[-1] = max(int(N[-1]), 256 - int(N[:-1].sum()) + 1) if K > 1 else max(int(N[0]), 300)
        r = rng.integers(20, 200, K).astype(np.int64)
        T = int(rng.integers(int(r.max()), int(r.max()) * 5))
        assert N.sum() > 255
        _check_table(P, N, r, T)


def test_dp_fill_long_rows_ragged(P, fillmode):
    # W = 71 (3 chunks of 32, ragged), small last size -> long in-row chains (J0 large)
    _check_table(P, np.array([5, 4, 70], np.int32), np.array([90, 70, 11], np.int64), 200)
    _check_table(P, np.array([3, 3, 3, 100], np.int32), np.array([50, 60, 70, 7], np.int64), 250)
    # J0 > 32: in-row chain crosses chunk boundaries
    _check_table(P, np.array([2, 120], np.int32), np.array([40, 3], np.int64), 150)
    # W = 33 and W = 32 exactly
    _check_table(P, np.array([6, 5, 32], np.int32), np.array([40, 50, 30], np.int64), 160)
    _check_table(P, np.array([6, 5, 31], np.int32), np.array([40, 50, 30], np.int64), 160)


def test_dp_fill_zero_counts_and_degenerate(P):
    _check_table(P, np.array([0, 3, 0, 4], np.int32), np.array([10, 20, 30, 40], np.int64), 60)
    opt, tab, st = P.dp_fill(np.zeros(0, np.int32), np.zeros(0, np.int64), 10)
    assert opt == 0 and tab.shape == () and int(tab) == 0
    opt, tab, st = P.dp_fill([0, 0], [5, 50], 10)   # sizes > T allowed when count is 0
    assert opt == 0
    _check_table(P, np.array([1], np.int32), np.array([7], np.int64), 7)
    _check_table(P, np.array([9], np.int32), np.array([7], np.int64), 7)   # one per machine


def test_dp_fill_invalid(P):
    with pytest.raises(P.PtasError) as ei:
        P.dp_fill([3], [11], 10)            # size > T with count > 0
    assert ei.value.rc == -1
    with pytest.raises(P.PtasError) as ei:
        P.dp_fill([-1], [5], 10)
    assert ei.value.rc == -1
    with pytest.raises(P.PtasError) as ei:
        P.dp_fill([40000, 40000], [5, 5], 10)   # sum N > 65535
    assert ei.value.rc == -2


@pytest.mark.parametrize("mode", ["1", "2"])
def test_dp_fill_scalar_kernel(P, monkeypatch, mode):
    # 1: the full-relaxation scalar kernel (fallback of the sharded compact path);
    # 2: the long-row two-launch path (row_cross + row_chain, rows > 1 KiB), forced
    # on every level, on the same random cases
    monkeypatch.setenv("PTAS_FORCE_SCALAR", mode)
    rng = np.random.default_rng(31)
    for K in (1, 2, 3, 5, 7):
        for _ in range(4):
            N, r, T = _rand_case(rng, K, {1: 200, 2: 60, 3: 25, 5: 8, 7: 4}[K])
            _check_table(P, N, r, T)
    _check_table(P, np.array([5, 4, 70], np.int32), np.array([90, 70, 11], np.int64), 200)


@pytest.mark.parametrize("split", ["0", "1000000000"])
def test_dp_fill_row_split_modes(P, monkeypatch, split):
    # small-level mode (8 warps share a row set) forced on / off for every level
    monkeypatch.setenv("PTAS_SPLIT_ROWS", split)
    monkeypatch.setenv("PTAS_DF", "0")   # one launch per row-level (the knob is theirs)
    rng = np.random.default_rng(57)
    for K in (2, 3, 5, 7):
        for _ in range(3):
            N, r, T = _rand_case(rng, K, {2: 60, 3: 25, 5: 8, 7: 4}[K])
            _check_table(P, N, r, T)
    _check_table(P, np.array([5, 4, 70], np.int32), np.array([90, 70, 11], np.int64), 200)
    _check_table(P, np.array([30, 40, 300], np.int32), np.array([90, 70, 11], np.int64), 200)


@pytest.mark.parametrize("ch", ["1", "2", "4", "8"])
def test_dp_fill_lane_layouts(P, monkeypatch, ch):
    # words per lane forced (group width Lg = ceil(words/CH), any value 1..32)
    monkeypatch.setenv("PTAS_SWAR_CH", ch)
    monkeypatch.setenv("PTAS_DF", "0")   # one launch per row-level (the knob is theirs)
    for W in (3, 5, 7, 13, 20, 29, 33, 61, 100, 127):
        _check_table(P, np.array([3, 4, W - 1], np.int32), np.array([35, 50, 21], np.int64), 110)
    rng = np.random.default_rng(int(ch))
    for K in (4, 6):
        for _ in range(3):
            N, r, T = _rand_case(rng, K, {4: 12, 6: 6}[K])
            _check_table(P, N, r, T)


def test_dp_fill_very_long_rows(P):
    # rows longer than 1 KiB (uint16, W = 701) use the long-row path; W*e = 1024 B exactly uses 8 chunks
    _check_table(P, np.array([2, 700], np.int32), np.array([60, 13], np.int64), 120)
    _check_table(P, np.array([3, 511], np.int32), np.array([60, 13], np.int64), 120)
    _check_table(P, np.array([1, 1, 300], np.int32), np.array([50, 40, 7], np.int64), 120)
    # long rows with ragged chunk tails, J0 > 32 (in-row source in an earlier chunk) and J0 = 1
    _check_table(P, np.array([4, 3, 1200], np.int32), np.array([300, 170, 3], np.int64), 310)
    _check_table(P, np.array([6, 1500], np.int32), np.array([100, 99], np.int64), 250)
    _check_table(P, np.array([2, 2, 2, 900], np.int32), np.array([40, 35, 33, 5], np.int64), 100)


def test_dp_fill_long_rows_solve(P):
    # a full solve whose DPs have rows > 1 KiB (N = [32, 1200], uint16 rows of 2402 B):
    # probe log, T*, makespan, assignment
    p = np.array([100] * 30 + [110] * 2 + [130] * 1200, np.int64)
    np.random.default_rng(0).shuffle(p)
    got = _cmp_solve(P, p, 420, 0.25, 1)
    assert max(x[5] for x in got["probes"]) == 39633


def test_dp_fill_padding_pitches(P, fillmode):
    # row byte lengths 1..9 (u8) and odd u16 lengths: every padding case of the packed kernel
    for W in range(1, 10):
        _check_table(P, np.array([4, 3, W - 1], np.int32), np.array([35, 50, 21], np.int64), 110)
    for W in (1, 2, 3, 5, 33, 65):
        _check_table(P, np.array([100, 150, W - 1], np.int32), np.array([35, 50, 21], np.int64), 110)


def test_dp_fill_device_torch(P):
    import torch
    N = np.array([7, 9, 40], np.int32)
    r = np.array([33, 45, 20], np.int64)
    sg, e = P.dp_table_shape(N)
    t = torch.full((sg,), 255, dtype=torch.uint8, device="cuda:0")
    s = torch.cuda.Stream()
    s.wait_stream(torch.cuda.current_stream())   # the fill above is ordered before the DP
    opt = P.dp_fill_device(N, r, 150, t, stream=s)
    want, _ = oracle.dp(N, r, 150)
    torch.cuda.synchronize()
    assert (t.cpu().numpy().reshape(want.shape).astype(np.int64) == want).all()
    assert opt == want[tuple(N)]


def test_dp_fill_two_word_packing(P, fillmode, monkeypatch):
    # force the leading digits into two 64-bit words (exercises the NW=2 kernels)
    monkeypatch.setenv("PTAS_FORCE_TWO_WORDS", "1")
    rng = np.random.default_rng(77)
    for K in (3, 5, 8):
        for _ in range(4):
            N, r, T = _rand_case(rng, K, {3: 20, 5: 6, 8: 3}[K])
            _check_table(P, N, r, T)


# ------------------------------------------------------------------ end to end
def _cmp_solve(P, p, m, eps, Pp, **kw):
    got = P.ptas_solve(p, m, eps, P=Pp, **kw)
    want = oracle.ptas(p, m, eps, Pp)
    assert got["T_star"] == want["T_star"]
    assert got["makespan"] == want["makespan"]
    assert got["assignment"].tolist() == want["assignment"].tolist()
    assert [(T, rd, f, K, o) for (T, rd, f, K, o, _s, _h) in got["probes"]] == \
           [(T, rd, f, K, o) for (T, rd, f, K, o, _s) in want["probes"]]
    return got


def test_solve_m1_seeds(P):
    for seed in range(120):
        p = jobs(12, 100, seed)
        for Pp in (1, 4):
            _cmp_solve(P, p, 3, 0.3, Pp)


def test_solve_layouts_and_memo(P):
    for seed in range(20):
        p = jobs(16, 100, seed)
        for layout in (0, 1):
            for memo in (True, False):
                _cmp_solve(P, p, 3, 0.25, 2, layout=layout, memoize=memo)


def test_solve_concurrent_probes_identical(P, monkeypatch):
    # P > 1 probes of a round run concurrently in separate DP slots; results and
    # the probe log must equal the sequential evaluation and the oracle
    for seed in range(6):
        p = jobs(60, 1000, seed)
        conc = _cmp_solve(P, p, 14, 0.3, 4)
        monkeypatch.setenv("PTAS_NO_CONCURRENT", "1")
        seq = P.ptas_solve(p, 14, 0.3, P=4)
        monkeypatch.delenv("PTAS_NO_CONCURRENT")
        assert seq["T_star"] == conc["T_star"] and (seq["assignment"] == conc["assignment"]).all()
        assert [x[:5] for x in seq["probes"]] == [x[:5] for x in conc["probes"]]
    p = jobs(40, 1000, 11)
    _cmp_solve(P, p, 8, 0.25, 8)   # 8 concurrent slots


def test_solve_g3_nonmonotone(P):
    g = json.load(open(os.path.join(GOLD, "g3_nonmonotone.json")))
    for Pp, want in g["by_P"].items():
        got = P.ptas_solve(g["p"], g["m"], g["eps"], P=int(Pp))
        assert got["T_star"] == want["T_star"] and got["makespan"] == want["makespan"]
        assert [[T, f] for (T, _r, f, *_x) in got["probes"]] == want["probes"]


def test_solve_g2(P):
    g = json.load(open(os.path.join(GOLD, "g2_m1_seed0.json")))
    got = P.ptas_solve(g["p"], g["m"], g["eps"], P=1)
    assert got["T_star"] == g["T_star"] and got["makespan"] == g["makespan"]
    assert got["assignment"].tolist() == g["assignment"]


def test_solve_medium_instances(P, fillmode):
    # shaped like the paper's workloads but small enough for the oracle
    for (n, m, eps, seed) in [(40, 8, 0.3, 1), (60, 14, 0.3, 2), (50, 10, 0.2, 3), (30, 5, 0.15, 4)]:
        p = jobs(n, 1000, seed)
        for Pp in (1, 3):
            _cmp_solve(P, p, m, eps, Pp)


def test_solve_virtual_shards_identical(P):
    for seed in range(6):
        p = jobs(40, 1000, seed)
        ref = P.ptas_solve(p, 8, 0.3, P=1)
        for vs in (2, 3, 8):
            got = P.ptas_solve(p, 8, 0.3, P=1, mode=P.MODE_LEVEL_SHARDED, virtual_shards=vs)
            assert got["T_star"] == ref["T_star"] and got["makespan"] == ref["makespan"]
            assert (got["assignment"] == ref["assignment"]).all()
            assert [x[:5] for x in got["probes"]] == [x[:5] for x in ref["probes"]]


def test_solve_empty_dp_literal(P):
    for name in ("M2", "M3", "M4"):
        w = WORKLOADS[name]
        got = P.ptas_solve(w.p(), w.m, w.eps, P=1)
        want = oracle.ptas(w.p(), w.m, w.eps, 1)
        assert got["T_star"] == want["T_star"] and got["makespan"] == want["makespan"]
        assert got["assignment"].tolist() == want["assignment"].tolist()


def test_solve_device_variant(P):
    import torch
    p = jobs(60, 1000, 9)
    pd = torch.from_numpy(p).cuda()
    # default stream: p produced by a kernel just before the call (legacy default stream order)
    pd = (pd * 2) // 2
    ad = torch.zeros(60, dtype=torch.int32, device="cuda")
    got = P.ptas_solve_device(pd, 14, 0.3, ad)
    want = oracle.ptas(p, 14, 0.3, 1)
    assert got["makespan"] == want["makespan"]
    assert ad.cpu().numpy().tolist() == want["assignment"].tolist()


def test_solve_invalid(P):
    for args in [([], 3, 0.3), ([1, 2], 0, 0.3), ([1, 0], 2, 0.3), ([1, 2], 2, 0.0), ([1, 2], 2, float("nan"))]:
        with pytest.raises(P.PtasError) as ei:
            P.ptas_solve(*args)
        assert ei.value.rc == -1


# ------------------------------------------------------------------ full size (bench configuration)
def _subbox(N, cap_sigma=2_000_000):
    Nc = N.copy()
    while np.prod(Nc.astype(np.float64) + 1) > cap_sigma:
        i = int(np.argmax(Nc))
        Nc[i] -= 1
    return Nc


@pytest.mark.parametrize("name", ["M2s", "M4s", "M3s"])
def test_full_size_dp_sampled(P, fillmode, name):
    """Full-size DP of the workload at T = LB (its largest probe): exact parity
    on a sub-box (the DP restricted to n <= N' equals the oracle's DP on N'),
    Eq. 1 re-checked at sampled states, and invariants on the whole table."""
    w = WORKLOADS[name]
    p = w.p()
    k = oracle.k_of(w.eps)
    LB, _ = oracle.bounds(p, w.m)
    u, r, N, _ = oracle.classify(p, LB, k)
    opt, tab, st = P.dp_fill(N, r, LB)
    t64 = tab.astype(np.int64)
    Nc = _subbox(N)
    want, _ = oracle.dp(Nc, r, LB)
    sub = t64[tuple(slice(0, int(x) + 1) for x in Nc)]
    assert (sub == want).all()
    C = oracle.configs(N, r, LB)
    assert st["relaxations"] == sum(float(np.prod((N - s + 1).astype(np.float64))) for s in C)
    rng = np.random.default_rng(0)
    for _ in range(3000):
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


# ------------------------------------------------------------------ speculative bisection (D8)
def test_speculation_preserves_alg1(P):
    """P = 1 with the next levels of the bisection tree evaluated concurrently:
    same probe log, T*, makespan and assignment as without speculation and as
    the oracle; the counted work is that of the probed DPs only."""
    cases = [(jobs(60, 1000, s), 14, 0.3) for s in range(4)] + [(jobs(12, 100, s), 3, 0.3) for s in range(20)]
    cases.append((WORKLOADS["M2s"].p(), WORKLOADS["M2s"].m, WORKLOADS["M2s"].eps))
    used = 0
    for p, m, eps in cases:
        ref = P.ptas_solve(p, m, eps, P=1, speculate=0)
        assert ref["stats"]["spec_dps"] == 0
        for d in (1, 2, 3, -1):   # -1: the default feasible-branch chain
            got = P.ptas_solve(p, m, eps, P=1, speculate=d)
            assert got["T_star"] == ref["T_star"] and got["makespan"] == ref["makespan"]
            assert (got["assignment"] == ref["assignment"]).all()
            assert got["probes"] == ref["probes"]   # incl. memo hits: speculation is not a memo hit
            st, rs = got["stats"], ref["stats"]
            assert st["relaxations"] == rs["relaxations"] and st["unique_dps"] == rs["unique_dps"]
            assert st["spec_wasted"] <= st["spec_dps"]
            used += st["spec_dps"]
        if len(p) <= 12:
            want = oracle.ptas(p, m, eps, 1)
            assert ref["T_star"] == want["T_star"] and ref["assignment"].tolist() == want["assignment"].tolist()
    assert used > 0


def test_fill_wall_time(P):
    """stats.fill_wall_seconds (union of the DPs' fill intervals): equal to the
    per-DP sum when DPs run one at a time, at most the sum (and at least the
    longest DP's fill) when speculative DPs overlap."""
    w = WORKLOADS["M2s"]
    for d in (0, 3):
        st = P.ptas_solve(w.p(), w.m, w.eps, P=1, speculate=d)["stats"]
        assert st["fill_wall_seconds"] > 0
        assert st["fill_wall_seconds"] <= st["fill_seconds"] * (1 + 1e-6) + 1e-6
        if d == 0:
            assert abs(st["fill_wall_seconds"] - st["fill_seconds"]) <= 0.02 * st["fill_seconds"] + 2e-5
    st = P.dp_fill(np.array([5, 4, 30], np.int32), np.array([60, 45, 17], np.int64), 160)[2]
    assert st["fill_wall_seconds"] == st["fill_seconds"]


@pytest.mark.parametrize("env", [{}, {"PTAS_ENUM_SYNC": "1"}, {"PTAS_NC_CAP": "5"}, {"PTAS_NP_CAP": "3"}])
def test_enumeration_without_round_trip(P, monkeypatch, env):
    """DPs after a slot's first are enqueued without reading |C| back (DESIGN.md
    D9): bit-exact tables on a sequence of DPs of varying size on one slot, with
    the bounds forced below |C| or the prefix count (every DP overflows, the
    kernels exit, the DP is redone synchronously) and with the synchronous path."""
    for k, v in env.items():
        monkeypatch.setenv(k, v)
    rng = np.random.default_rng(91)
    for it in range(14):
        K = int(rng.integers(2, 7))
        N, r, T = _rand_case(rng, K, {2: 40, 3: 20, 4: 9, 5: 6, 6: 4}[K])
        _check_table(P, N, r, T)
    for seed in range(6):
        _cmp_solve(P, jobs(40, 1000, seed), 8, 0.3, 1)


@pytest.mark.parametrize("domtab", ["0", "1"])
def test_dominance_table_modes(P, monkeypatch, domtab):
    """Per-row dominance masks from the DP's digit-threshold table (DESIGN.md
    D10, forced on for every K, uint8) or from the lane-parallel packed-digit
    test (forced off): bit-exact tables either way, in per-level and dataflow
    launches, including two-word digit packing."""
    monkeypatch.setenv("PTAS_DOMTAB", domtab)
    rng = np.random.default_rng(4242)
    for K in (2, 3, 5, 7, 9):
        for _ in range(3):
            N, r, T = _rand_case(rng, K, {2: 60, 3: 25, 5: 8, 7: 4, 9: 3}[K])
            _check_table(P, N, r, T)
    monkeypatch.setenv("PTAS_DF", "0")
    monkeypatch.setenv("PTAS_FORCE_TWO_WORDS", "1")
    for K in (3, 6):
        N, r, T = _rand_case(rng, K, {3: 20, 6: 5}[K])
        _check_table(P, N, r, T)


def test_hmbp_parity(P):
    """High-multiplicity bin packing (include/ptas.h hmbp_solve):
    bin count and packing identical to oracle.hmbp (same R11 traceback) on
    random instances incl. zero counts, uint16 tables and K = 1; a valid
    packing with the load bound at a larger size."""
    rng = np.random.default_rng(808)
    for it in range(40):
        K = int(rng.integers(1, 7))
        N = rng.integers(0, {1: 300, 2: 40, 3: 16, 4: 8, 5: 5, 6: 4}[K], K).astype(np.int32)
        if it % 5 == 0:
            N[rng.integers(0, K)] = 0
        if N.sum() == 0:
            N[0] = 3
        r = rng.integers(5, 100, K).astype(np.int64)
        T = int(rng.integers(int(r.max()), int(r.max()) * 4))
        bins, pk, st = P.hmbp_solve(N, r, T)
        wb, wpk = oracle.hmbp(N, r, T)
        assert bins == wb and pk.tolist() == wpk.tolist(), (N, r, T)
        assert st["kernel_launches"] > 0
    assert P.hmbp_solve([0, 0], [3, 4], 10)[0] == 0
    with pytest.raises(P.PtasError):
        P.hmbp_solve([1], [11], 10)
    # larger instance: validity + load bound (no oracle call on the full size)
    N = np.array([30, 25, 17, 20, 19, 13], np.int32)
    r = np.array([244, 355, 423, 511, 592, 677], np.int64)
    bins, pk, _ = P.hmbp_solve(N, r, 1674)
    assert (pk.sum(axis=0) == N).all() and ((pk * r).sum(axis=1) <= 1674).all()
    assert bins >= -(-int((N * r).sum()) // 1674)
    assert bins == P.dp_fill(N, r, 1674, table=False)[0]


@pytest.mark.parametrize("tb", ["0", "1", "reg0"])
def test_traceback_kernels(P, monkeypatch, tb):
    """Register traceback (default for |C| <= 64, K <= 12), warp traceback
    (configurations in shared memory, PTAS_TB_REG=0) and the block kernel:
    identical schedules, equal to the oracle's (reading R11)."""
    if tb == "reg0":
        monkeypatch.setenv("PTAS_TB_REG", "0")
    else:
        monkeypatch.setenv("PTAS_TB_BLOCK", tb)
    for seed in range(12):
        _cmp_solve(P, jobs(12, 100, seed), 3, 0.3, 1)
    for (n, m, eps, seed) in [(40, 8, 0.3, 1), (60, 14, 0.3, 2), (50, 10, 0.2, 3)]:
        _cmp_solve(P, jobs(n, 1000, seed), m, eps, 1)
    rng = np.random.default_rng(99)
    for _ in range(6):
        K = int(rng.integers(2, 6))
        N = rng.integers(1, 9, K).astype(np.int32)
        r = rng.integers(5, 80, K).astype(np.int64)
        T = int(rng.integers(int(r.max()), int(r.max()) * 3))
        bins, pk, _ = P.hmbp_solve(N, r, T)
        wb, wpk = oracle.hmbp(N, r, T)
        assert bins == wb and pk.tolist() == wpk.tolist()


@pytest.mark.parametrize("name", ["M4x", "M3g"])
def test_full_size_dp_sampled_device(P, name):
    """The two largest tables (M4x: K = 8, 1.75 GB uint8; M3g: 5.5 GB uint16)
    filled on the device at T = LB in the bench's launch configuration and
    checked there: exact parity with the oracle on a sub-box, Eq. 1 re-checked
    at 4000 sampled states (all configurations gathered at once), OPT(0) = 0,
    OPT(N) = the returned value, and monotonicity / +1 Lipschitz along every
    axis over the whole table (on the GPU)."""
    import torch
    w = WORKLOADS[name]
    p = w.p()
    k = oracle.k_of(w.eps)
    LB, _ = oracle.bounds(p, w.m)
    u, r, N, _ = oracle.classify(p, LB, k)
    N = np.asarray(N, np.int64)
    sg, e = P.dp_table_shape(N)
    t = torch.empty(sg, dtype=torch.uint8 if e == 1 else torch.int16, device="cuda:0")
    opt = P.dp_fill_device(N.astype(np.int32), r, LB, t)
    torch.cuda.synchronize()
    shape = tuple(int(x) + 1 for x in N)
    stride = np.ones(len(N), np.int64)
    for i in range(len(N) - 2, -1, -1):
        stride[i] = stride[i + 1] * shape[i + 1]
    tv = t.view(shape)

    def at(idx):   # int64 flat indices -> values (host)
        return t[torch.as_tensor(idx, device="cuda:0")].to(torch.int64).cpu().numpy() & (0xff if e == 1 else 0xffff)

    # sub-box parity
    Nc = _subbox(N, cap_sigma=150000)
    want, _ = oracle.dp(Nc, r, LB)
    grids = np.meshgrid(*[np.arange(int(x) + 1) for x in Nc], indexing="ij")
    flat = sum(g.astype(np.int64) * s for g, s in zip(grids, stride))
    assert (at(flat.ravel()).reshape(want.shape) == want).all()
    # Eq. 1 at sampled states
    C = oracle.configs(N, r, LB).astype(np.int64)
    off = C @ stride
    rng = np.random.default_rng(5)
    ns = np.stack([rng.integers(0, int(x) + 1, 4000) for x in N], axis=1)
    ns = ns[ns.any(axis=1)]
    idx = ns @ stride
    dom = (C[None, :, :] <= ns[:, None, :]).all(axis=2)          # [samples, |C|]
    src = np.where(dom, idx[:, None] - off[None, :], 0)
    vals = at(src.ravel()).reshape(src.shape)
    best = np.where(dom, vals, 1 << 30).min(axis=1)
    assert (at(idx) == best + 1).all()
    assert at(np.array([0]))[0] == 0 and opt == at(np.array([int(N @ stride)]))[0]
    # monotone and +1 Lipschitz along every axis (whole table, on the GPU)
    for ax in range(len(N)):
        a = tv.narrow(ax, 1, shape[ax] - 1).to(torch.int32)
        b = tv.narrow(ax, 0, shape[ax] - 1).to(torch.int32)
        d = a - b
        assert int(d.min()) >= 0 and int(d.max()) <= 1
        del a, b, d


@pytest.mark.parametrize("k", [4, 5, 7])
def test_dstar_shapes_full_table(P, k):
    # the D* roofline-sweep geometry (synth.dstar) at sizes the
    # oracle finishes in seconds: every entry vs the oracle, K = 3..8
    from synth import dstar
    for K in range(3, 9):
        N, r, T = dstar(K, 3.0e4 if k < 7 else 1.2e4, k)
        _check_table(P, N, r, T)


@pytest.mark.parametrize("vs", [2, 3, 8])
def test_virtual_shards_use_packed_kernel(P, vs):
    # sharded row-levels must keep the packed kernel (16-byte aligned compact slices):
    # identical results to the single-GPU solve AND the collapsed executed count
    w = WORKLOADS["M2s"]
    p = w.p()
    ref = P.ptas_solve(p, w.m, w.eps, P=1, speculate=0)
    got = P.ptas_solve(p, w.m, w.eps, P=1, mode=P.MODE_LEVEL_SHARDED, virtual_shards=vs, speculate=0)
    assert got["T_star"] == ref["T_star"] and got["makespan"] == ref["makespan"]
    assert (got["assignment"] == ref["assignment"]).all()
    assert got["stats"]["relaxations"] == ref["stats"]["relaxations"]
    assert got["stats"]["relax_executed"] == ref["stats"]["relax_executed"] < got["stats"]["relaxations"]


def test_long_row_path(P, monkeypatch):
    # long-row path (one warp per 4 chunks of 32 entries, pivot blocks, row 0 in
    # closed form) forced on every level; J0 from 1 to > 32
    monkeypatch.setenv("PTAS_FORCE_SCALAR", "2")
    _check_table(P, np.array([4, 3, 1200], np.int32), np.array([300, 170, 3], np.int64), 310)
    _check_table(P, np.array([6, 1500], np.int32), np.array([100, 99], np.int64), 250)
    _check_table(P, np.array([3, 3, 200], np.int32), np.array([50, 45, 1], np.int64), 60)
    rng = np.random.default_rng(77)
    for K in (2, 3, 4):
        for _ in range(3):
            N, r, T = _rand_case(rng, K, {2: 120, 3: 30, 4: 10}[K])
            _check_table(P, N, r, T)

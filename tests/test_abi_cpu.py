"""C-ABI checks that need no GPU: the library loads, exports every symbol the
header declares, validates arguments before touching CUDA, and its host-side
steps (classification, bounds, probe targets, interval update) agree with the
oracle bit for bit."""
from __future__ import annotations

import os
import re

import numpy as np
import pytest

import oracle
from synth import jobs

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


@pytest.fixture(scope="module")
def P():
    import paper_conf_ipps_ligsg18_b200 as P
    from paper_conf_ipps_ligsg18_b200 import build
    build.build()
    return P


def _header_functions():
    src = open(os.path.join(ROOT, "include", "ptas.h")).read()
    src = re.sub(r"/\*.*?\*/", "", src, flags=re.S)
    return sorted(set(re.findall(r"^\s*(?:const\s+)?\w+\s*\*?\s*(\w+)\s*\(", src, flags=re.M)))


def test_exports_every_header_symbol(P):
    names = _header_functions()
    assert "ptas_solve" in names and "dp_fill" in names and len(names) >= 19
    L = P.lib()
    for nm in names:
        assert hasattr(L, nm), nm
    assert sorted(P.EXPORTS) == names


def test_strerror(P):
    for rc in range(0, -7, -1):
        assert P.strerror(rc) and P.strerror(rc) != "unknown status"


def test_k_matches_oracle(P):
    for eps in [0.3, 0.2, 0.15, 0.25, 0.1, 0.5, 1.0, 0.33, 0.0999, 0.07]:
        assert P.ptas_k(eps) == oracle.k_of(eps)
    with pytest.raises(P.PtasError):
        P.ptas_k(0.0)


def test_bounds_match_oracle(P):
    for seed in range(50):
        p = jobs(int(np.random.default_rng(seed).integers(1, 300)), 1000, seed)
        for m in (1, 3, 17):
            assert P.ptas_bounds(p, m) == oracle.bounds(p, m)


def test_classify_matches_oracle(P):
    rng = np.random.default_rng(4)
    for seed in range(300):
        n = int(rng.integers(1, 200))
        p = jobs(n, int(rng.integers(2, 2000)), seed)
        k = int(rng.integers(1, 9))
        LB, UB = oracle.bounds(p, int(rng.integers(1, 40)))
        T = int(rng.integers(max(1, LB // 3), UB + 1))
        a = P.ptas_classify(p, T, k)
        b = oracle.classify(p, T, k)
        assert a[0] == b[0]
        assert a[1].tolist() == b[1].tolist() and a[2].tolist() == b[2].tolist()
        assert a[3].tolist() == b[3].tolist()


def test_search_steps_reproduce_oracle_probe_log(P):
    """Drive the search with the library's host steps and the oracle's DP as the
    feasibility test: the probe sequence must equal the oracle's own."""
    for seed in range(40):
        p = jobs(12, 100, seed)
        m, eps = 3, 0.3
        k = oracle.k_of(eps)
        for Pp in (1, 2, 3, 4, 8):
            LB, UB = P.ptas_bounds(p, m)
            seq = []
            while LB < UB:
                Ts = P.ptas_probe_targets(LB, UB, Pp)
                f = []
                for T in Ts:
                    u, r, N, _ = oracle.classify(p, T, k)
                    opt = int(oracle.dp(N, r, T)[0][tuple(N)]) if len(N) else 0
                    f.append(int(opt <= m))
                    seq.append((T, f[-1]))
                LB, UB = P.ptas_interval_update(LB, UB, Ts, f)
            want = oracle.ptas(p, m, eps, Pp)
            assert seq == [(T, fe) for (T, _r, fe, *_x) in want["probes"]]
            assert LB == want["T_star"]


def test_shard_range_partition(P):
    for count in (0, 1, 7, 100, 1001):
        for world in (1, 2, 3, 8):
            spans = [P.ptas_shard_range(count, r, world) for r in range(world)]
            covered = [i for b, e in spans for i in range(b, e)]
            assert covered == list(range(count))


def test_invalid_arguments_rejected_before_cuda(P):
    # validation happens before any CUDA call, so these are EINVAL even without a GPU
    with pytest.raises(P.PtasError) as ei:
        P.ptas_solve([1, 0, 3], 2, 0.3)
    assert ei.value.rc == -1
    with pytest.raises(P.PtasError) as ei:
        P.ptas_solve([1, 2, 3], 0, 0.3)
    assert ei.value.rc == -1
    with pytest.raises(P.PtasError) as ei:
        P.ptas_solve([1, 2, 3], 2, -1.0)
    assert ei.value.rc == -1
    with pytest.raises(P.PtasError) as ei:
        P.dp_fill([2, 3], [5, 50], 10)
    assert ei.value.rc == -1
    with pytest.raises(P.PtasError) as ei:
        P.dp_table_shape([2**31 - 1] * 3)
    assert ei.value.rc == -2
    assert P.dp_table_shape([3, 0, 4]) == (20, 1)
    assert P.dp_table_shape([200, 100]) == (201 * 101, 2)


def test_no_cpu_fallback_in_product():
    """The product package never imports the oracle."""
    pkg = os.path.join(ROOT, "paper_conf_ipps_ligsg18_b200")
    for dp, _dn, fns in os.walk(pkg):
        for fn in fns:
            if fn.endswith((".py", ".cpp", ".cu", ".h")):
                src = open(os.path.join(dp, fn)).read()
                assert "import oracle" not in src and "from oracle" not in src and "ptas_oracle" not in src, fn


def test_table_order_rule(P):
    # layout 0 (D2/D13): non-empty classes only, the largest count last
    # (ties: the highest index), the others by descending size; layout 1: given order
    assert P.ptas_table_order([30, 25, 17, 20, 19, 13], [416, 520, 624, 728, 832, 936]) == [5, 4, 3, 2, 1, 0]
    got = P.ptas_table_order([3, 0, 7, 7], [10, 20, 30, 40])
    assert got[-1] == 3 and sorted(got) == [0, 2, 3] and got[:2] == [2, 0]
    assert P.ptas_table_order([3, 0, 7, 7], [10, 20, 30, 40], layout=1) == [0, 2, 3]
    assert P.ptas_table_order([0, 0], [5, 6]) == []
    rng = np.random.default_rng(7)
    for _ in range(50):
        K = int(rng.integers(1, 9))
        N = rng.integers(0, 20, K)
        r = rng.permutation(np.arange(1, K + 1) * 10)
        o = P.ptas_table_order(N, r)
        nz = [i for i in range(K) if N[i] > 0]
        assert sorted(o) == nz
        if nz:
            assert N[o[-1]] == max(N[nz])
            lead = o[:-1]
            assert all(r[lead[i]] > r[lead[i + 1]] for i in range(len(lead) - 1))


def test_level_shard_split(P):
    # the engine's split of a row-level (ptas_level_shard): aligned slices that tile [0, R)
    rng = np.random.default_rng(11)
    for _ in range(200):
        R = int(rng.integers(0, 5000))
        W = int(rng.integers(1, 8))
        rb = int(rng.integers(1, 700))
        cover = []
        for g in range(W):
            b, e, ch = P.ptas_level_shard(R, g, W, rb)
            assert (ch * rb) % 16 == 0 and ch >= -(-R // W) if R else True
            assert 0 <= b <= e <= R and (e == b or b == g * ch)
            cover += list(range(b, e))
        assert cover == list(range(R))
    for bad in [(-1, 0, 1, 1), (5, 1, 1, 1), (5, 0, 0, 1), (5, 0, 1, 0)]:
        with pytest.raises(P.PtasError):
            P.ptas_level_shard(*bad)

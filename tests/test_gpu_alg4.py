"""The paper's own DP design (Alg 4 / Alg 5 data partitioning)
rebuilt as an A/B baseline (csrc/alg4.cu): every table entry
equals the oracle's, for several partition dimensions `dim` (the paper used
3..9), uint8 and uint16 tables, and the divisor follows Alg 4 l.4-10."""
from __future__ import annotations

import math

import numpy as np
import pytest

import oracle

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def P():
    import paper_conf_ipps_ligsg18_b200 as P
    return P


def _divisor(N, dim):
    d = []
    for n in N:
        v = int(math.floor(math.sqrt(n + 1)))
        while v > 1 and (n + 1) % v:
            v -= 1
        d.append(max(v, 1))
    keep = sorted(range(len(N)), key=lambda i: -d[i])[:dim]   # stable: ties by index
    return [d[i] if i in keep else 1 for i in range(len(N))]


@pytest.mark.parametrize("dim", [1, 3, 6, 9])
def test_alg4_tables_vs_oracle(P, dim):
    rng = np.random.default_rng(400 + dim)
    for it in range(12):
        K = int(rng.integers(2, 7))
        N = rng.integers(1, {2: 60, 3: 25, 4: 12, 5: 8, 6: 6}[K], K).astype(np.int32)
        if it % 4 == 0:
            N[rng.integers(0, K)] += 255
        r = rng.integers(20, 200, K).astype(np.int64)
        T = int(rng.integers(int(r.max()), int(r.max()) * 4))
        opt, tab, div, st = P.dp_fill_alg4(N, r, T, dim=dim)
        want, relax = oracle.dp(N, r, T)
        assert (tab.astype(np.int64) == want).all(), (N.tolist(), r.tolist(), T, dim)
        assert opt == int(want[tuple(N)]) and st["relaxations"] == relax
        assert div == _divisor(N.tolist(), dim)


def test_alg4_paper_example_shape(P):
    # Fig. 2's 6 x 6 x 6 table (the figure divides it by (3, 3, 3); Alg 4's own rule,
    # l.6-8, gives floor(sqrt(6)) = 2, which divides 6: 8 blocks of 3 x 3 x 3, 4 block-levels)
    N = np.array([5, 5, 5], np.int32)
    r = np.array([30, 40, 50], np.int64)
    opt, tab, div, st = P.dp_fill_alg4(N, r, 120, dim=3)
    assert div == [2, 2, 2] and st["fill_launches"] == 4
    want, _ = oracle.dp(N, r, 120)
    assert (tab.astype(np.int64) == want).all()

"""K = 3 cluster ring kernel (row_ring.cu, D14) against the oracle,
entry by entry: 1 to 4 row-levels per cluster barrier (temporal blocking with
redundant rows below each CTA's block), every cluster size, uint8 and uint16
tables, one- and two-word windows.  A case counts only when the ring kernel
actually filled it (one fill launch for the whole DP)."""
from __future__ import annotations

import numpy as np
import pytest

import oracle

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def P():
    import paper_conf_ipps_ligsg18_b200 as lib
    lib.lib()
    return lib


def _case(rng, e):
    while True:
        if e == 1:
            N = rng.integers(2, 40, 3).astype(np.int32)
            N[0] = rng.integers(32, 100)       # A = ceil((N0 + 1) / 16) >= hi0 at every cluster size
            N[2] = rng.integers(4, 120)
            if N.sum() > 255:
                continue
        else:
            N = rng.integers(20, 120, 3).astype(np.int32)
            N[2] = rng.integers(60, 300)
            if N.sum() <= 255:
                continue
        r = np.sort(rng.integers(30, 300, 3))[::-1].astype(np.int64)   # row class smallest: J0 >= 1
        T = int(rng.integers(int(r[0]), int(r[0]) * 4))
        if min(int(N[2]), T // int(r[2])) * e > 8:     # the ring kernel's window limit
            continue
        return N, r, T


@pytest.mark.parametrize("e", [1, 2])
@pytest.mark.parametrize("tb", ["1", "2", "3", "4"])
@pytest.mark.parametrize("cs", ["2", "4", "8", "16"])
def test_ring_temporal_blocking_vs_oracle(P, monkeypatch, e, tb, cs):
    monkeypatch.setenv("PTAS_RING_TB", tb)
    monkeypatch.setenv("PTAS_RING_SMEM_TARGET", str(220 * 1024))   # the requested TB wherever it fits
    monkeypatch.setenv("PTAS_RING_CS", cs)
    rng = np.random.default_rng(7000 + 10 * e + int(cs))
    used = 0
    for _ in range(8):
        N, r, T = _case(rng, e)
        opt, tab, st = P.dp_fill(N, r, T)
        want, relax = oracle.dp(N, r, T)
        bad = np.argwhere(tab.astype(np.int64) != want)
        assert len(bad) == 0, (N.tolist(), r.tolist(), T, bad[:5].tolist())
        assert opt == int(want[tuple(N)])
        assert st["relaxations"] == relax
        used += st["fill_launches"] == 1
    assert used >= 4, "ring kernel rarely taken: %d of 8 cases" % used

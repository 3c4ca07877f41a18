"""Bit-exact parity on the BASELINE-shaped workloads themselves (SURVEY.md §8(d)
M2s, M3s, M3g, M4s, M4x, M5s-0.3/0.2/0.15) — the configurations bench.py times.

* Whole solves (Alg 1 / Alg 3) through the C ABI in
  the bench's launch configuration: probe log (T, round, feasible, K, OPT(N),
  sigma), T*, makespan and assignment equal the oracle's, from the goldens in
  tests/golden/shaped/ (written by scripts/make_shaped_goldens.py, which calls
  only oracle/) and, for M5s-0.3 and M5s-0.2, from a live oracle run.
* The largest DP table of every workload (T = LB) in the SOLVE's internal
  layout (ptas_table_order, D2/D13): every entry of Eq. 1
   equals the oracle's — entry by entry against a live oracle
  run for M2s, M3s, M5s-0.3 and M5s-0.2, through the SHA-256 of the whole table
  (in the oracle's class order) for all of them incl. M3g (5.5 GB) and M4x.
"""
from __future__ import annotations

import glob
import hashlib
import json
import os

import numpy as np
import pytest

import oracle
from synth import WORKLOADS

pytestmark = pytest.mark.gpu
GOLD = os.path.join(os.path.dirname(__file__), "golden", "shaped")


def _solve_goldens():
    out = []
    for f in sorted(glob.glob(os.path.join(GOLD, "solve_*.json"))):
        g = json.load(open(f))
        out.append(pytest.param(g, id=f"{g['workload']}-P{g['P']}"))
    return out


def _table_goldens():
    return [pytest.param(json.load(open(f)), id=json.load(open(f))["workload"])
            for f in sorted(glob.glob(os.path.join(GOLD, "table_*.json")))]


@pytest.fixture(scope="module")
def P():
    import paper_conf_ipps_ligsg18_b200 as P
    return P


def _cmp(got, want):
    assert got["T_star"] == want["T_star"]
    assert got["makespan"] == want["makespan"]
    assert [int(x) for x in got["assignment"]] == [int(x) for x in want["assignment"]]
    assert [list(x[:6]) for x in got["probes"]] == [list(x) for x in want["probes"]]


@pytest.mark.parametrize("g", _solve_goldens())
def test_shaped_solve_matches_oracle_golden(P, g):
    w = WORKLOADS[g["workload"]]
    assert (w.n, w.m, w.eps, w.P, w.seed) == (g["n"], g["m"], g["eps"], g["P_jobs"], g["seed"])
    _cmp(P.ptas_solve(w.p(), w.m, w.eps, P=g["P"]), g)


@pytest.mark.parametrize("name", ["M5s-0.3", "M5s-0.2"])
def test_shaped_solve_live_oracle(P, name):
    w = WORKLOADS[name]
    want = oracle.ptas(w.p(), w.m, w.eps, 1)
    _cmp(P.ptas_solve(w.p(), w.m, w.eps, P=1), want)


def _solve_layout_table_device(P, g):
    """The workload's largest DP filled on the device in the solve's internal
    layout; returns (torch tensor viewed in the ORACLE's class order, opt, order)."""
    import torch
    N = np.asarray(g["N"], np.int32)
    r = np.asarray(g["r"], np.int64)
    order = P.ptas_table_order(N, r, 0)
    assert sorted(order) == list(range(len(N)))
    No, ro = N[order], r[order]
    sg, e = P.dp_table_shape(No)
    assert sg == g["sigma"] and e == g["e"]
    t = torch.empty(sg, dtype=torch.uint8 if e == 1 else torch.int16, device="cuda:0")
    opt = P.dp_fill_device(No, ro, g["T"], t)
    torch.cuda.synchronize()
    inv = np.argsort(order)          # internal axis of each oracle class
    tv = t.view(tuple(int(x) + 1 for x in No)).permute(*[int(i) for i in inv])
    return tv, opt, order


def _sha256_device(tv):
    """SHA-256 of a (permuted) device tensor's bytes in row-major order, streamed
    to the host in slabs along axis 0."""
    h = hashlib.sha256()
    n0 = tv.shape[0]
    step = max(1, int((256 << 20) // max(1, tv[0].numel() * tv.element_size())))
    for a in range(0, n0, step):
        h.update(tv[a:a + step].contiguous().cpu().numpy().tobytes())
    return h.hexdigest()


@pytest.mark.parametrize("g", _table_goldens())
def test_shaped_table_sha256_solve_layout(P, g):
    w = WORKLOADS[g["workload"]]
    k = P.ptas_k(w.eps)
    LB, _ = P.ptas_bounds(w.p(), w.m)
    u, r, N, _ = P.ptas_classify(w.p(), LB, k)
    assert LB == g["T"] and N.tolist() == g["N"] and r.tolist() == g["r"]
    tv, opt, _ = _solve_layout_table_device(P, g)
    assert opt == g["opt"]
    for q, v in g["samples"]:
        assert int(tv[tuple(q)]) & (0xff if g["e"] == 1 else 0xffff) == v
    assert _sha256_device(tv) == g["sha256"]


@pytest.mark.parametrize("name", ["M2s", "M3s", "M5s-0.3", "M5s-0.2"])
def test_shaped_table_every_entry_live_oracle(P, name):
    w = WORKLOADS[name]
    k = oracle.k_of(w.eps)
    LB, _ = oracle.bounds(w.p(), w.m)
    u, r, N, _ = oracle.classify(w.p(), LB, k)
    want, relax = oracle.dp(N, r, LB)
    g = {"N": N.tolist(), "r": r.tolist(), "T": LB, "sigma": int(want.size), "e": 1 if N.sum() <= 255 else 2}
    tv, opt, order = _solve_layout_table_device(P, g)
    got = tv.contiguous().cpu().numpy().astype(np.int64) & (0xff if g["e"] == 1 else 0xffff)
    bad = np.argwhere(got != want)
    assert len(bad) == 0, bad[:5].tolist()
    assert opt == int(want[tuple(N)])
    # the executed-relaxation count and the closed form over the solve's own DP
    st = P.ptas_solve(w.p(), w.m, w.eps, P=1)["stats"]
    assert st["relaxations"] > 0 and st["relax_executed"] < st["relaxations"]

"""Multi-process (gloo, world_size 2, CPU) checks of the N>1 host logic.

The GPU data path of both multi-GPU modes cannot run here; what is covered is
the protocol each rank executes around it, with the library's own host steps:

* multi-section search (MULTI_PROBE, Alg 3 generalised):
  every rank derives the same probe list with ptas_probe_targets, evaluates
  only probe j == rank (here with the oracle's DP: test infrastructure),
  exchanges OPT(N) with an all-gather, and applies ptas_interval_update.  The
  result must equal the single-process oracle run with P = world.
* level sharding (LEVEL_SHARDED): each rank takes the
  engine's aligned slice (ptas_level_shard) of every row-level, "computes" it
  (row ids), the slices are all-gathered with the equal-count padding the
  engine uses, and the scattered result must cover every row exactly once.
"""
from __future__ import annotations

import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def _free_port():
    with socket.socket() as s:
        s.bind(("127.0.0.1", 0))
        return s.getsockname()[1]


def _worker(rank, world, port, fn, q):
    import sys
    sys.path.insert(0, ROOT)
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        q.put((rank, fn(rank, world)))
    except Exception as e:  # pragma: no cover - surfaced by the parent
        q.put((rank, repr(e)))
    finally:
        dist.destroy_process_group()


def _run(fn, world=2):
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    ps = [ctx.Process(target=_worker, args=(r, world, port, fn, q)) for r in range(world)]
    for p in ps:
        p.start()
    out = dict(q.get(timeout=300) for _ in ps)
    for p in ps:
        p.join(timeout=60)
    return [out[r] for r in range(world)]


def multisection_rank(rank, world):
    import oracle
    import paper_conf_ipps_ligsg18_b200 as P
    from synth import jobs
    results = []
    for seed in range(12):
        p = jobs(12, 100, seed)
        m, eps = 3, 0.3
        k = P.ptas_k(eps)
        LB, UB = P.ptas_bounds(p, m)
        seq = []
        while LB < UB:
            Ts = P.ptas_probe_targets(LB, UB, world)
            mine = -1
            if rank < len(Ts):
                u, r, N, _ = oracle.classify(p, Ts[rank], k)
                mine = int(oracle.dp(N, r, Ts[rank])[0][tuple(N)]) if len(N) else 0
            allv = [torch.zeros(1, dtype=torch.int32) for _ in range(world)]
            dist.all_gather(allv, torch.tensor([mine], dtype=torch.int32))
            opts = [int(t.item()) for t in allv][: len(Ts)]
            f = [int(o <= m) for o in opts]
            seq += list(zip(Ts, f))
            LB, UB = P.ptas_interval_update(LB, UB, Ts, f)
        want = oracle.ptas(p, m, eps, world)
        results.append((seq == [(T, fe) for (T, _r, fe, *_x) in want["probes"]], LB == want["T_star"]))
    return results


def sharding_rank(rank, world):
    """The engine's own split of a row-level (ptas_level_shard, dp_engine.cpp): rank
    g fills rows [b, e) of the level into its compact slice of `chunk` rows of
    row_bytes bytes (16-byte aligned, padded to equal counts), the slices are
    all-gathered in rank order, and the scatter reads slot s at s * row_bytes:
    every row must arrive exactly once, from its owner."""
    import paper_conf_ipps_ligsg18_b200 as P
    rng = np.random.default_rng(3)
    ok = True
    for _ in range(40):
        R = int(rng.integers(1, 500))
        row_bytes = int(rng.integers(1, 80))
        b, e, chunk = P.ptas_level_shard(R, rank, world, row_bytes)
        ok &= (chunk * row_bytes) % 16 == 0 and chunk >= -(-R // world)
        ok &= b == min(R, rank * chunk) and e == min(R, b + chunk)
        mine = torch.full((chunk * row_bytes,), -1, dtype=torch.int64)
        for s in range(b, e):
            mine[(s - b) * row_bytes:(s - b + 1) * row_bytes] = s
        gathered = [torch.empty(chunk * row_bytes, dtype=torch.int64) for _ in range(world)]
        dist.all_gather(gathered, mine)
        flat = torch.cat(gathered)
        for s in range(R):
            ok &= bool((flat[s * row_bytes:(s + 1) * row_bytes] == s).all())
    return ok


@pytest.mark.timeout(600)
def test_multisection_protocol_gloo():
    res = _run(multisection_rank, 2)
    for r in res:
        assert not isinstance(r, str), r
        assert all(a and b for a, b in r)
    assert res[0] == res[1]


@pytest.mark.timeout(600)
def test_level_shard_gather_scatter_gloo():
    res = _run(sharding_rank, 2)
    assert res == [True, True]


# ---- slab/halo pipeline (ptas_options.slab_pipeline): the
# engine's schedule with the library's own plan (ptas_slab_plan).  Per chunk,
# rank g receives the halo slabs from g - 1 (gloo send/recv in place of
# ncclSend/ncclRecv, carrying the slab ids), "fills" its slabs in ascending
# order -- asserting that every slab a row reads (p0 - s0, 1 <= s0 <= hi0, at the
# same or an earlier chunk) is present -- and forwards its last hout slabs.
def _pipeline_protocol(rank, world):
    import paper_conf_ipps_ligsg18_b200 as P
    out = []
    for S, hi0, C in [(251, 2, 8), (31, 4, 5), (7, 3, 3), (world, 5, 2), (120, 0, 4)]:
        pb, pe, pbase, hin, hout = P.ptas_slab_plan(S, hi0, rank, world)
        have = set()
        for c in range(C):
            if rank > 0 and hin > 0:
                t = torch.zeros(hin, dtype=torch.int64)
                dist.recv(t, src=rank - 1)
                got = sorted(int(x) for x in t)
                assert got == list(range(pb - hin, pb)), (S, hi0, rank, c, got)
                have.update((s, c) for s in got)
            for p0 in range(pb, pe):
                for s0 in range(1, hi0 + 1):
                    if p0 - s0 >= 0:
                        assert p0 - s0 >= pbase, (S, hi0, rank, p0, s0)
                        assert all((p0 - s0, cc) in have for cc in range(c + 1)), (S, hi0, rank, p0, s0, c)
                have.add((p0, c))
            if rank + 1 < world and hout > 0:
                ids = list(range(pe - hout, pe))
                assert all((s, c) in have for s in ids)
                dist.send(torch.tensor(ids, dtype=torch.int64), dst=rank + 1)
        out.append((pb, pe, pbase, hin, hout))
    return out


@pytest.mark.parametrize("world", [2, 3])
def test_slab_pipeline_protocol(world):
    res = _run(_pipeline_protocol, world)
    for k, (S, hi0) in enumerate([(251, 2), (31, 4), (7, 3), (world, 5), (120, 0)]):
        plans = [r[k] for r in res]
        # contiguous, disjoint, covering ranges; the last rank owns slab S - 1 (OPT(N))
        assert plans[0][0] == 0 and plans[-1][1] == S
        for g in range(1, world):
            assert plans[g][0] == plans[g - 1][1]
            assert plans[g][3] == plans[g - 1][4]          # hin(g) == hout(g - 1)
        assert all(p[1] > p[0] for p in plans)

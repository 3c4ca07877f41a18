"""The real NCCL code path on the one GPU a round has: a world-size-1 NCCL
communicator created through torch.distributed (unique-id broadcast) drives

* LEVEL_SHARDED with shard_min_rows = 0: EVERY row-level goes through the
  sharded path -- fill of the rank's aligned slice (ptas_level_shard) into the
  compact stage buffer, ncclAllGather, row_scatter into the table -- plus the
  admission agreement (ncclAllReduce of the status word) before the first
  collective;
* MULTI_PROBE: per-round OPT(N) exchange (ncclAllGather) and the traceback on
  the owning rank with its machine configurations broadcast (ncclBroadcast).

Results are compared with the ORACLE (goldens written by
scripts/make_shaped_goldens.py from oracle/ only, and live oracle runs), not
with the single-GPU solve."""
from __future__ import annotations

import json
import os
import socket

import pytest

import oracle
from synth import WORKLOADS, jobs

pytestmark = pytest.mark.gpu
GOLD = os.path.join(os.path.dirname(__file__), "golden", "shaped")


def _port():
    with socket.socket() as s:
        s.bind(("127.0.0.1", 0))
        return s.getsockname()[1]


@pytest.fixture(scope="module")
def comm():
    import torch
    import torch.distributed as dist
    import paper_conf_ipps_ligsg18_b200 as P
    os.environ.setdefault("MASTER_ADDR", "127.0.0.1")
    os.environ["MASTER_PORT"] = str(_port())
    torch.cuda.set_device(0)
    dist.init_process_group("nccl", rank=0, world_size=1, device_id=torch.device("cuda:0"))
    c = P.init_comm(0)
    yield P, c
    c.destroy()
    dist.destroy_process_group()


def _cmp(got, want):
    assert got["T_star"] == want["T_star"]
    assert got["makespan"] == want["makespan"]
    assert [int(x) for x in got["assignment"]] == [int(x) for x in want["assignment"]]
    assert [list(x[:6]) for x in got["probes"]] == [list(x) for x in want["probes"]]


def test_level_sharded_every_level_nccl_vs_oracle(comm):
    P, c = comm
    for seed, (n, m, eps) in enumerate([(60, 14, 0.3), (40, 8, 0.25), (50, 10, 0.2)]):
        p = jobs(n, 1000, seed + 2)
        got = P.ptas_solve(p, m, eps, P=1, mode=P.MODE_LEVEL_SHARDED, comm=c, shard_min_rows=0)
        _cmp(got, oracle.ptas(p, m, eps, 1))
        assert got["stats"]["fill_launches"] > 0


@pytest.mark.parametrize("name", ["M2s", "M5s-0.3"])
def test_level_sharded_shaped_nccl_vs_golden(comm, name):
    P, c = comm
    w = WORKLOADS[name]
    g = json.load(open(os.path.join(GOLD, f"solve_{name}_P1.json")))
    _cmp(P.ptas_solve(w.p(), w.m, w.eps, P=1, mode=P.MODE_LEVEL_SHARDED, comm=c, shard_min_rows=0), g)


def test_level_sharded_default_threshold_nccl(comm):
    # default threshold (2048 rows): small levels redundant, large ones sharded
    P, c = comm
    w = WORKLOADS["M2s"]
    g = json.load(open(os.path.join(GOLD, "solve_M2s_P1.json")))
    _cmp(P.ptas_solve(w.p(), w.m, w.eps, P=1, mode=P.MODE_LEVEL_SHARDED, comm=c), g)


def test_multi_probe_nccl_vs_oracle(comm):
    P, c = comm
    for seed in range(4):
        p = jobs(40, 1000, seed)
        _cmp(P.ptas_solve(p, 8, 0.3, P=1, mode=P.MODE_MULTI_PROBE, comm=c), oracle.ptas(p, 8, 0.3, 1))
    w = WORKLOADS["M5s-0.2"]
    g = json.load(open(os.path.join(GOLD, "solve_M5s-0.2_P1.json")))
    _cmp(P.ptas_solve(w.p(), w.m, w.eps, P=1, mode=P.MODE_MULTI_PROBE, comm=c), g)


def test_level_shard_split_exported(comm):
    # the exported split is the one the engine uses: aligned, covering, rank 0 owns all at world 1
    P, _ = comm
    for R, rb in [(1, 1), (7, 31), (2048, 17), (12345, 612)]:
        b, e, ch = P.ptas_level_shard(R, 0, 1, rb)
        assert (b, e) == (0, R) and (ch * rb) % 16 == 0 and ch >= R


@pytest.mark.parametrize("name", ["M2s", "M5s-0.3"])
def test_window_slabs_sharded_nccl_vs_golden(comm, name):
    """Level window + level sharding: every probe DP keeps only
    min(N0, T/r0) + 1 slabs, and every slab (and every level of slab 0) goes through
    the rank slice -> ncclAllGather -> scatter path; the schedule's DP at T* is full."""
    P, c = comm
    w = WORKLOADS[name]
    g = json.load(open(os.path.join(GOLD, f"solve_{name}_P1.json")))
    got = P.ptas_solve(w.p(), w.m, w.eps, P=1, mode=P.MODE_LEVEL_SHARDED, comm=c, shard_min_rows=0, window=1)
    _cmp(got, g)
    assert got["stats"]["window_dps"] > 0


@pytest.mark.parametrize("name", ["M2s", "M5s-0.3", "M3s"])
def test_slab_pipeline_nccl_vs_golden(comm, name):
    """Slab/halo pipeline (ptas_options.slab_pipeline): every
    probe DP is filled in chunks of the other classes' levels, slab by slab, in the
    rank's linear slab buffer (at world size 1 the rank owns every slab and there is
    no halo to send); OPT(N) is read on the last rank and broadcast.  The probe log,
    T*, makespan and assignment equal the oracle's."""
    P, c = comm
    w = WORKLOADS[name]
    g = json.load(open(os.path.join(GOLD, f"solve_{name}_P1.json")))
    got = P.ptas_solve(w.p(), w.m, w.eps, P=1, mode=P.MODE_LEVEL_SHARDED, comm=c, window=1, slab_pipeline=1)
    _cmp(got, g)
    assert got["stats"]["window_dps"] > 0


@pytest.mark.parametrize("chunks", ["1", "4", "64"])
def test_slab_pipeline_random_vs_oracle(comm, monkeypatch, chunks):
    # chunks per rank (1: the whole slab at once; 64: one level per chunk for small DPs)
    P, c = comm
    monkeypatch.setenv("PTAS_PIPE_CHUNKS_PER_RANK", chunks)
    for seed, (n, m, eps) in enumerate([(60, 14, 0.3), (40, 8, 0.25), (50, 10, 0.2), (30, 9, 0.34)]):
        p = jobs(n, 1000, seed + 11)
        got = P.ptas_solve(p, m, eps, P=1, mode=P.MODE_LEVEL_SHARDED, comm=c, window=1, slab_pipeline=1)
        _cmp(got, oracle.ptas(p, m, eps, 1))

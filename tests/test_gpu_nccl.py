"""The real NCCL code path on the one GPU a round has: a world-size-1 NCCL
communicator created through torch.distributed (unique-id broadcast) drives
the LEVEL_SHARDED mode (per-row-level compact slice -> ncclAllGather ->
scatter) and the MULTI_PROBE mode (per-round OPT(N) exchange).  Results must
equal the single-GPU solve bit for bit (determinism across modes, §8(b))."""
from __future__ import annotations

import os
import socket

import pytest

from synth import jobs

pytestmark = pytest.mark.gpu


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


def test_level_sharded_nccl_world1(comm):
    P, c = comm
    for seed, (n, m, eps) in enumerate([(60, 14, 0.3), (40, 8, 0.25), (200, 60, 0.3)]):
        p = jobs(n, 1000, seed + 2)
        ref = P.ptas_solve(p, m, eps, P=1)
        got = P.ptas_solve(p, m, eps, P=1, mode=P.MODE_LEVEL_SHARDED, comm=c)
        assert got["T_star"] == ref["T_star"] and got["makespan"] == ref["makespan"]
        assert (got["assignment"] == ref["assignment"]).all()
        assert [x[:5] for x in got["probes"]] == [x[:5] for x in ref["probes"]]


def test_multi_probe_nccl_world1(comm):
    P, c = comm
    for seed in range(4):
        p = jobs(40, 1000, seed)
        ref = P.ptas_solve(p, 8, 0.3, P=1)
        got = P.ptas_solve(p, 8, 0.3, P=1, mode=P.MODE_MULTI_PROBE, comm=c)
        assert got["T_star"] == ref["T_star"] and got["makespan"] == ref["makespan"]
        assert (got["assignment"] == ref["assignment"]).all()

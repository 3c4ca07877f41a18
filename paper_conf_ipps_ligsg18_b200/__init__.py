"""B200-native PTAS for P||Cmax (Li, Ghalami, Schwiebert, Grosu, IPDPS-W 2018).

Python binding of ``libptas_b200.so`` with the names of the C ABI
(``include/ptas.h``).  Marshalling only; PyTorch is used for device memory,
streams and process groups.  See DESIGN.md.
"""
from __future__ import annotations

import ctypes

import numpy as np

from ._native import (MODE_LEVEL_SHARDED, MODE_MULTI_PROBE, MODE_SINGLE, EXPORTS, PtasError, PtasOptions,
                      PtasProbe, PtasStats, _a, _chk, _ptr, lib, strerror)

__all__ = ["ptas_solve", "ptas_solve_device", "dp_fill", "dp_fill_opt", "dp_fill_alg4", "dp_fill_device", "hmbp_solve", "dp_table_shape", "dp_configs",
           "dp_row_index", "ptas_k", "ptas_bounds", "ptas_classify", "ptas_probe_targets",
           "ptas_interval_update", "ptas_shard_range", "ptas_level_shard", "ptas_table_order", "Comm", "init_comm", "options", "lib", "strerror",
           "PtasError", "EXPORTS", "MODE_SINGLE", "MODE_LEVEL_SHARDED", "MODE_MULTI_PROBE"]


def options(P: int = 1, mode: int = MODE_SINGLE, device: int = -1, comm=None, budget: int = 0,
            memoize: bool = True, virtual_shards: int = 1, layout: int = 0, stream=None,
            speculate: int = -1, shard_min_rows: int = -1, window: int = 0, slab_pipeline: int = 0) -> PtasOptions:
    o = PtasOptions()
    lib().ptas_default_options(ctypes.byref(o))
    o.probes_per_round = int(P)
    o.mode = int(mode)
    o.device = int(device)
    o.comm = comm.handle if comm is not None else None
    o.table_budget_bytes = int(budget)
    o.memoize = int(bool(memoize))
    o.virtual_shards = int(virtual_shards)
    o.layout = int(layout)
    o.speculate = int(speculate)
    o.shard_min_rows = int(shard_min_rows)
    o.window = int(window)
    o.slab_pipeline = int(slab_pipeline)
    o.stream = None if stream is None else ctypes.c_void_p(stream.cuda_stream if hasattr(stream, "cuda_stream") else int(stream))
    return o


def ptas_solve(p, m: int, eps: float, P: int = 1, log: bool = True, opts: PtasOptions | None = None, **kw):
    """PTAS of Alg 1/3 with the GPU DP.  Returns dict(makespan, assignment, T_star, stats, probes)."""
    p = _a(p, np.int64)
    n = len(p)
    o = opts if opts is not None else options(P=P, **kw)
    ms = ctypes.c_int64()
    asg = np.zeros(n, np.int32)
    st = PtasStats()
    cap = 4096
    plog = (PtasProbe * cap)()
    nlog = ctypes.c_int32()
    rc = lib().ptas_solve_ex(_ptr(p, ctypes.c_int64), n, int(m), float(eps), ctypes.byref(o), ctypes.byref(ms),
                             _ptr(asg, ctypes.c_int32), ctypes.byref(st), plog if log else None,
                             cap if log else 0, ctypes.byref(nlog))
    _chk("ptas_solve", rc)
    probes = [(plog[i].T, plog[i].round, plog[i].feasible, plog[i].K, plog[i].opt, plog[i].sigma,
               plog[i].memo_hit) for i in range(min(nlog.value, cap))] if log else []
    return {"makespan": ms.value, "assignment": asg, "T_star": st.T_star, "stats": st.to_dict(), "probes": probes}


def ptas_solve_device(p_dev, m: int, eps: float, assignment_dev, P: int = 1, opts: PtasOptions | None = None, **kw):
    """Device-resident variant: p_dev (int64) and assignment_dev (int32) are CUDA tensors."""
    import torch
    assert p_dev.is_cuda and p_dev.dtype == torch.int64 and p_dev.is_contiguous()
    assert assignment_dev.is_cuda and assignment_dev.dtype == torch.int32 and assignment_dev.numel() == p_dev.numel()
    if opts is None and "stream" not in kw:
        # the caller's current stream: p_dev is read after the work that produced it
        kw["stream"] = torch.cuda.current_stream(p_dev.device)
    o = opts if opts is not None else options(P=P, device=p_dev.device.index, **kw)
    ms = ctypes.c_int64()
    st = PtasStats()
    rc = lib().ptas_solve_device(ctypes.c_void_p(p_dev.data_ptr()), p_dev.numel(), int(m), float(eps),
                                 ctypes.byref(o), ctypes.byref(ms), ctypes.c_void_p(assignment_dev.data_ptr()),
                                 ctypes.byref(st))
    _chk("ptas_solve_device", rc)
    return {"makespan": ms.value, "T_star": st.T_star, "stats": st.to_dict()}


def dp_table_shape(counts):
    c = _a(counts, np.int32)
    sg, e = ctypes.c_int64(), ctypes.c_int32()
    _chk("dp_table_shape", lib().dp_table_shape(_ptr(c, ctypes.c_int32), len(c), ctypes.byref(sg), ctypes.byref(e)))
    return sg.value, e.value


def dp_fill(counts, sizes, T: int, table: bool = True):
    """Whole OPT table (host ndarray, row-major over the given class order) and OPT(N)."""
    c = _a(counts, np.int32)
    s = _a(sizes, np.int64)
    sg, e = dp_table_shape(c)
    out = np.zeros(sg, np.uint8 if e == 1 else np.uint16) if table else None
    opt = ctypes.c_int32()
    st = PtasStats()
    rc = lib().dp_fill(_ptr(c, ctypes.c_int32), _ptr(s, ctypes.c_int64), len(c), int(T),
                       out.ctypes.data_as(ctypes.c_void_p) if table else None, sg * e if table else 0,
                       ctypes.byref(opt), ctypes.byref(st))
    _chk("dp_fill", rc)
    if table:
        out = out.reshape(tuple(int(x) + 1 for x in c)) if len(c) else out.reshape(())
    return opt.value, out, st.to_dict()


def dp_fill_opt(counts, sizes, T: int, budget: int = 0, window: int = 0):
    """OPT(N) only, with the level window when the table exceeds `budget` bytes
    (window=1: always, -1: never).  Returns (opt, stats)."""
    c = _a(counts, np.int32)
    s = _a(sizes, np.int64)
    opt = ctypes.c_int32()
    st = PtasStats()
    _chk("dp_fill_opt", lib().dp_fill_opt(_ptr(c, ctypes.c_int32), _ptr(s, ctypes.c_int64), len(c), int(T),
                                          int(budget), int(window), ctypes.byref(opt), ctypes.byref(st)))
    return opt.value, st.to_dict()


def dp_fill_alg4(counts, sizes, T: int, dim: int = 6, table: bool = True):
    """The paper's Alg 4 partitioned DP (A/B baseline): (opt, table or None, divisor, stats)."""
    c = _a(counts, np.int32)
    s = _a(sizes, np.int64)
    sg, e = dp_table_shape(c)
    out = np.zeros(sg, np.uint8 if e == 1 else np.uint16) if table else None
    opt = ctypes.c_int32()
    dv = np.zeros(max(len(c), 1), np.int32)
    st = PtasStats()
    _chk("dp_fill_alg4", lib().dp_fill_alg4(_ptr(c, ctypes.c_int32), _ptr(s, ctypes.c_int64), len(c), int(T), int(dim),
                                            out.ctypes.data_as(ctypes.c_void_p) if table else None,
                                            sg * e if table else 0, ctypes.byref(opt), _ptr(dv, ctypes.c_int32),
                                            ctypes.byref(st)))
    if table:
        out = out.reshape(tuple(int(x) + 1 for x in c))
    return opt.value, out, dv[: len(c)].tolist(), st.to_dict()


def hmbp_solve(counts, sizes, capacity: int, packing: bool = True):
    """High-multiplicity bin packing on the level-fill engine (include/ptas.h):
    (bins, packing[bins, K] int32 or None, stats)."""
    c = _a(counts, np.int32)
    s = _a(sizes, np.int64)
    K = len(c)
    mx = max(int(c.sum()), 1)
    pk = np.zeros((mx, max(K, 1)), np.int32) if packing else None
    bins = ctypes.c_int32()
    st = PtasStats()
    rc = lib().hmbp_solve(_ptr(c, ctypes.c_int32), _ptr(s, ctypes.c_int64), K, int(capacity), ctypes.byref(bins),
                          pk.ctypes.data_as(ctypes.POINTER(ctypes.c_int32)) if packing else None, mx,
                          ctypes.byref(st))
    _chk("hmbp_solve", rc)
    return bins.value, (pk[:bins.value, :K].copy() if packing else None), st.to_dict()


def dp_fill_device(counts, sizes, T: int, table_dev, stream=None) -> int:
    """Fill a caller-owned CUDA tensor (uint8/uint16, >= sigma entries) on `stream`."""
    import torch
    c = _a(counts, np.int32)
    s = _a(sizes, np.int64)
    if stream is None:
        stream = torch.cuda.current_stream(table_dev.device)
    opt = ctypes.c_int32()
    rc = lib().dp_fill_device(_ptr(c, ctypes.c_int32), _ptr(s, ctypes.c_int64), len(c), int(T),
                              ctypes.c_void_p(table_dev.data_ptr()), table_dev.numel() * table_dev.element_size(),
                              ctypes.c_void_p(stream.cuda_stream), ctypes.byref(opt))
    _chk("dp_fill_device", rc)
    return opt.value


def dp_configs(counts, sizes, T: int) -> np.ndarray:
    c = _a(counts, np.int32)
    s = _a(sizes, np.int64)
    K = len(c)
    cnt = ctypes.c_int64()
    _chk("dp_configs", lib().dp_configs(_ptr(c, ctypes.c_int32), _ptr(s, ctypes.c_int64), K, int(T), None, 0,
                                        ctypes.byref(cnt)))
    out = np.zeros(max(cnt.value * K, 1), np.int32)
    _chk("dp_configs", lib().dp_configs(_ptr(c, ctypes.c_int32), _ptr(s, ctypes.c_int64), K, int(T),
                                        _ptr(out, ctypes.c_int32), cnt.value, ctypes.byref(cnt)))
    return out[: cnt.value * K].reshape(cnt.value, K)


def dp_row_index(counts):
    """(level_start[rho_max+2], rowbase[rows]) of the row-level index."""
    c = _a(counts, np.int32)
    sg, _ = dp_table_shape(c)
    nz = c[c > 0]
    W = int(nz[-1]) + 1 if len(nz) else 1
    rho_max = int(nz[:-1].sum()) if len(nz) else 0
    ls = np.zeros(rho_max + 2, np.int64)
    rb = np.zeros(max(sg // W, 1), np.int64)
    _chk("dp_row_index", lib().dp_row_index(_ptr(c, ctypes.c_int32), len(c), _ptr(ls, ctypes.c_int64), len(ls),
                                            _ptr(rb, ctypes.c_int64), len(rb)))
    return ls, rb


# ------------------------------------------------------------ host steps (no GPU)
def ptas_k(eps: float) -> int:
    k = lib().ptas_k(float(eps))
    _chk("ptas_k", 0 if k > 0 else k)
    return k


def ptas_bounds(p, m: int):
    p = _a(p, np.int64)
    lb, ub = ctypes.c_int64(), ctypes.c_int64()
    _chk("ptas_bounds", lib().ptas_bounds(_ptr(p, ctypes.c_int64), len(p), int(m), ctypes.byref(lb), ctypes.byref(ub)))
    return lb.value, ub.value


def ptas_classify(p, T: int, k: int):
    p = _a(p, np.int64)
    n = len(p)
    u, K = ctypes.c_int64(), ctypes.c_int32()
    r = np.zeros(n, np.int64)
    N = np.zeros(n, np.int32)
    cls = np.zeros(n, np.int32)
    _chk("ptas_classify", lib().ptas_classify(_ptr(p, ctypes.c_int64), n, int(T), int(k), ctypes.byref(u),
                                              ctypes.byref(K), _ptr(r, ctypes.c_int64), _ptr(N, ctypes.c_int32),
                                              _ptr(cls, ctypes.c_int32)))
    return u.value, r[: K.value].copy(), N[: K.value].copy(), cls


def ptas_probe_targets(LB: int, UB: int, P: int):
    out = np.zeros(P, np.int64)
    cnt = ctypes.c_int32()
    _chk("ptas_probe_targets", lib().ptas_probe_targets(int(LB), int(UB), int(P), _ptr(out, ctypes.c_int64),
                                                        ctypes.byref(cnt)))
    return [int(x) for x in out[: cnt.value]]


def ptas_interval_update(LB: int, UB: int, T, feasible):
    T = _a(T, np.int64)
    f = _a(feasible, np.int32)
    lb, ub = ctypes.c_int64(LB), ctypes.c_int64(UB)
    _chk("ptas_interval_update", lib().ptas_interval_update(ctypes.byref(lb), ctypes.byref(ub),
                                                            _ptr(T, ctypes.c_int64), _ptr(f, ctypes.c_int32), len(T)))
    return lb.value, ub.value


def ptas_table_order(counts, sizes, layout: int = 0):
    """Internal class order of the DP table (list of caller class indices, non-empty classes)."""
    c = _a(counts, np.int32)
    s = _a(sizes, np.int64)
    out = np.zeros(max(len(c), 1), np.int32)
    k = ctypes.c_int32()
    _chk("ptas_table_order", lib().ptas_table_order(_ptr(c, ctypes.c_int32), _ptr(s, ctypes.c_int64), len(c),
                                                    int(layout), _ptr(out, ctypes.c_int32), ctypes.byref(k)))
    return [int(x) for x in out[: k.value]]


def ptas_slab_plan(S: int, hi0: int, rank: int, world: int):
    """(pb, pe, pbase, hin, hout) of the slab/halo pipeline (ptas_options.slab_pipeline)."""
    v = [ctypes.c_int64() for _ in range(5)]
    _chk("ptas_slab_plan", lib().ptas_slab_plan(int(S), int(hi0), int(rank), int(world), *[ctypes.byref(x) for x in v]))
    return tuple(x.value for x in v)


def ptas_level_shard(rows: int, rank: int, world: int, row_bytes: int):
    """(begin, end, chunk) of the level-sharded DP's aligned split of one row-level."""
    b, e, c = ctypes.c_int64(), ctypes.c_int64(), ctypes.c_int64()
    _chk("ptas_level_shard", lib().ptas_level_shard(int(rows), int(rank), int(world), int(row_bytes), ctypes.byref(b),
                                                    ctypes.byref(e), ctypes.byref(c)))
    return b.value, e.value, c.value


def ptas_shard_range(count: int, rank: int, world: int):
    b, e = ctypes.c_int64(), ctypes.c_int64()
    _chk("ptas_shard_range", lib().ptas_shard_range(int(count), int(rank), int(world), ctypes.byref(b), ctypes.byref(e)))
    return b.value, e.value


# ------------------------------------------------------------ multi-GPU
class Comm:
    """NCCL communicator owned by the library; created collectively."""

    def __init__(self, handle, rank, world):
        self.handle = handle
        self.rank = rank
        self.world = world

    def destroy(self):
        if self.handle:
            lib().ptas_comm_destroy(self.handle)
            self.handle = None


def init_comm(device: int | None = None) -> Comm:
    """Collective over the default torch.distributed group: rank 0 makes the
    NCCL unique id, torch broadcasts it, every rank joins."""
    import torch
    import torch.distributed as dist
    rank, world = dist.get_rank(), dist.get_world_size()
    if device is None:
        device = torch.cuda.current_device()
    buf = (ctypes.c_uint8 * 128)()
    if rank == 0:
        _chk("ptas_get_unique_id", lib().ptas_get_unique_id(ctypes.cast(buf, ctypes.c_void_p)))
    t = torch.tensor(list(bytes(buf)), dtype=torch.uint8,
                     device=f"cuda:{device}" if dist.get_backend() == "nccl" else "cpu")
    dist.broadcast(t, 0)
    raw = bytes(t.cpu().tolist())
    ctypes.memmove(buf, raw, 128)
    h = ctypes.c_void_p()
    _chk("ptas_comm_init", lib().ptas_comm_init(ctypes.byref(h), rank, world, ctypes.cast(buf, ctypes.c_void_p), device))
    return Comm(h, rank, world)

#!/usr/bin/env python3
"""Benchmark of the PTAS hot path (BASELINE.json metric: DP state-relaxations/sec
and PTAS solve time; %HBM peak).

One step = one full ptas_solve of the workload (every §8(a) row: classify,
configuration enumeration, row-level index, level fill per probe, readout,
search, traceback + greedy schedule).

  python bench.py [--gpus N] [--steps K] [--warmup W] [--workload W] [--impl ours|reference]

Workloads: N = 1 -> M2s (the shaped twin of configs[1], the
single-GPU level-fill baseline); N > 1 -> M4x level-sharded (north_star's
largest-dimension instance, configs[3]'s role), with a multi-section block on
M5s-0.3 at P = N (configs[4]).  The N = 1 line carries the single-GPU M4x
number in `scaling_ref` so every N of a scaling run has the same instance.

value  : Eq. 1 relaxations (closed form, summed over the DPs the search used;
         speculative DPs the search never probed are not counted) / device-timed
         step, with p resident in HBM (ptas_solve_device)
e2e    : the same through ptas_solve with pinned host p / host assignment
roofline: level fill, SURVEY.md §8(d) algorithmic bytes (relax + sigma) * e over
         the fill time (CUDA events: union of the DPs' fill intervals) against
         N x MEASURED_PEAKS.json hbm_gbs.  The kernels gather fewer bytes than
         Eq. 1 (one window per prefix, pivot blocks, D5/D13), so
         frac > 1 is possible; `frac_executed` uses the bytes actually gathered
         and `dram` the ncu DRAM bytes of the profiled launch (profiles/).
parity : asserted on every run, outside the timed region: the solve (T*,
         makespan, assignment, probe log) against the oracle's golden
         (tests/golden/shaped, written by scripts/make_shaped_goldens.py from
         oracle/ only) and the SHA-256 of the largest DP table (T = LB) in the
         solve's layout against the oracle's.  A mismatch exits non-zero.
cpu_baseline: the oracle (plain sequential C) on the workload's largest DP (the
         whole table when it is at most 6e9 relaxations, else a sub-box), one
         host core; cpu_baseline.omp: the paper's Alg 2 comparator shape (OpenMP
         level-parallel) on all host cores, same table
"""
from __future__ import annotations

import argparse
import json
import os
import statistics
import sys
import threading
import time

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)
# load every kernel of the library at context creation: lazy loading would put
# module loads of the fill-kernel variants inside the first timed steps
os.environ.setdefault("CUDA_MODULE_LOADING", "EAGER")

import numpy as np  # noqa: E402

from synth import WORKLOADS  # noqa: E402

METRIC = "DP state-relaxations/sec and PTAS solve time at 1/2/4/8 B200; %HBM peak"
UNIT = "relaxations/s"


def _peaks():
    try:
        with open(os.path.join(ROOT, "MEASURED_PEAKS.json")) as f:
            d = json.load(f)
        return float(d["hbm_gbs"]), "measured"
    except Exception:
        return 6650.0, "fallback"


class ClockSampler:
    """SM clock and throttle reasons sampled in-process through NVML during the
    timed region (no nvidia-smi subprocesses, which stall the driver)."""

    def __init__(self, index: int, period: float = float(os.environ.get("BENCH_CLOCK_PERIOD", "0.01"))):
        self.index = index
        self.period = period
        self.rows = []
        self._stop = threading.Event()
        self._t = threading.Thread(target=self._run, daemon=True)
        self.err = None

    def _run(self):
        try:
            import pynvml as nv
            nv.nvmlInit()
            h = nv.nvmlDeviceGetHandleByIndex(self.index)
            mx = nv.nvmlDeviceGetMaxClockInfo(h, nv.NVML_CLOCK_SM)
            while not self._stop.is_set():
                sm = nv.nvmlDeviceGetClockInfo(h, nv.NVML_CLOCK_SM)
                rs = nv.nvmlDeviceGetCurrentClocksEventReasons(h) if hasattr(nv, "nvmlDeviceGetCurrentClocksEventReasons") \
                    else nv.nvmlDeviceGetCurrentClocksThrottleReasons(h)
                self.rows.append((sm, mx, rs))
                self._stop.wait(self.period)
        except Exception as e:  # pragma: no cover - reported in the JSON line
            self.err = repr(e)

    def __enter__(self):
        if os.environ.get("BENCH_NO_CLOCKS") != "1":
            self._t.start()
        return self

    def __exit__(self, *a):
        self._stop.set()
        if self._t.is_alive():
            self._t.join(timeout=10)

    def summary(self):
        if not self.rows:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["unsampled"], "error": self.err}
        bits = {0x8: "hw_slowdown", 0x40: "hw_thermal_slowdown", 0x20: "sw_thermal_slowdown",
                0x4: "sw_power_cap", 0x80: "hw_power_brake_slowdown"}
        reasons = set()
        for _sm, _mx, rs in self.rows:
            for b, nm in bits.items():
                if rs & b:
                    reasons.add(nm)
        return {"sm_mhz": statistics.median(r[0] for r in self.rows), "sm_max_mhz": max(r[1] for r in self.rows),
                "reasons": sorted(reasons), "samples": len(self.rows)}


def _dist_env():
    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    return rank, local, world


def _largest_dp(w):
    """(N, r, T) of the workload's DP at T = LB — the largest table of the solve."""
    import oracle
    p = w.p()
    k = oracle.k_of(w.eps)
    LB, _ = oracle.bounds(p, w.m)
    u, r, N, _ = oracle.classify(p, LB, k)
    return N, r, LB


def _largest_dp_product(w):
    """(N, r, T) at T = LB through the library's exported host steps (no oracle)."""
    import paper_conf_ipps_ligsg18_b200 as P
    p = w.p()
    k = P.ptas_k(w.eps)
    LB, _ = P.ptas_bounds(p, w.m)
    _u, r, N, _ = P.ptas_classify(p, LB, k)
    return N, r, LB


def _subbox_for(N, r, T, target_relax):
    """Clip counts (largest first) until the closed-form relaxation count of the
    sub-box DP is <= target: the DP restricted to n <= N' is exactly the
    oracle's DP on N' (same C(T) restricted), so it is a sample of the same
    workload."""
    import oracle
    C = oracle.configs(N, r, T)
    Nc = np.array(N, np.int64)

    def relax(Nv):
        ok = (C <= Nv).all(axis=1)
        return float(np.prod((Nv - C[ok] + 1).astype(np.float64), axis=1).sum())
    while relax(Nc) > target_relax and Nc.max() > 1:
        i = int(np.argmax(Nc))
        Nc[i] -= 1
    return Nc.astype(np.int32), relax(Nc)


def _cpu_model():
    try:
        for line in open("/proc/cpuinfo"):
            if line.startswith("model name"):
                return line.split(":", 1)[1].strip()
    except OSError:
        pass
    return None


def cpu_oracle_sample(w, target_relax=6.0e9):
    """The oracle on the workload's largest DP (T = LB): the whole table when its
    closed-form relaxation count is at most target_relax, else a sub-box."""
    import oracle
    N, r, T = _largest_dp(w)
    if len(N) == 0:
        return None
    Nc, rel = _subbox_for(N, r, T, target_relax)
    whole = bool((np.asarray(Nc) == np.asarray(N)).all())
    t0 = time.perf_counter()
    _tab, relax = oracle.dp(Nc, r, T)
    dt = time.perf_counter() - t0
    what = (f"oracle_dp on the WHOLE {w.name} DP at T=LB={T} (N={list(map(int, N))})" if whole else
            f"oracle_dp on the sub-box N'={Nc.tolist()} of the {w.name} DP at T=LB={T} (full N={list(map(int, N))})")
    out = {"value": relax / dt, "unit": UNIT, "cores": 1, "kind": "oracle", "cpu_model": _cpu_model(),
           "nproc": os.cpu_count(), "whole_table": whole,
           "sample": f"{what}; {relax:.3g} relaxations in {dt:.2f} s, 1 core"}
    # The paper's comparator shape (Alg 2, OpenMP level-parallel) on all host
    # cores, same table; its table must equal the sequential oracle's.
    try:
        t0 = time.perf_counter()
        tab2, relax2 = oracle.dp_omp(Nc, r, T)
        dt2 = time.perf_counter() - t0
        cores = oracle.omp_threads()
        out["omp"] = {"value": relax2 / dt2, "unit": UNIT, "cores": cores, "kind": "oracle_alg2_openmp",
                      "tables_equal": bool(np.array_equal(_tab, tab2)),
                      "sample": f"oracle_dp_omp (Alg 2 level-parallel) on the same table; "
                                f"{relax2:.3g} relaxations in {dt2:.2f} s, {cores} threads"}
    except Exception as e:  # noqa: BLE001 — the comparator is optional context
        out["omp"] = {"unavailable": str(e)}
    return out


GOLD = os.path.join(ROOT, "tests", "golden", "shaped")


def parity_check(P, w, opts, Pp, table=True):
    """Bit-exact parity of this run's configuration against the oracle's goldens
    (tests/golden/shaped): the solve, and the largest DP table in the solve's
    layout.  Returns a dict; raises SystemExit on a mismatch."""
    import hashlib
    import torch
    out = {}
    p = w.p()
    gs = os.path.join(GOLD, f"solve_{w.name}_P{Pp}.json")
    if os.path.exists(gs):
        g = json.load(open(gs))
        got = P.ptas_solve(p, w.m, w.eps, opts=opts, log=True)
        ok = (got["T_star"] == g["T_star"] and got["makespan"] == g["makespan"] and
              [int(x) for x in got["assignment"]] == g["assignment"] and
              [list(x[:6]) for x in got["probes"]] == g["probes"])
        out["solve"] = {"match": ok, "T_star": got["T_star"], "makespan": got["makespan"],
                        "probes": len(got["probes"]), "golden": os.path.relpath(gs, ROOT)}
    else:
        out["solve"] = {"match": None, "note": f"no oracle golden for {w.name} at P={Pp}"}
    gt = os.path.join(GOLD, f"table_{w.name}.json")
    if table and os.path.exists(gt):
        g = json.load(open(gt))
        N = np.asarray(g["N"], np.int32)
        r = np.asarray(g["r"], np.int64)
        order = P.ptas_table_order(N, r, 0)
        No, ro = N[order], r[order]
        sg, e = P.dp_table_shape(No)
        t = torch.empty(sg, dtype=torch.uint8 if e == 1 else torch.int16, device=torch.cuda.current_device())
        opt = P.dp_fill_device(No, ro, g["T"], t)
        torch.cuda.synchronize()
        tv = t.view(tuple(int(x) + 1 for x in No)).permute(*[int(i) for i in np.argsort(order)])
        h = hashlib.sha256()
        step = max(1, int((256 << 20) // max(1, tv[0].numel() * tv.element_size())))
        for a in range(0, tv.shape[0], step):
            h.update(tv[a:a + step].contiguous().cpu().numpy().tobytes())
        ok = h.hexdigest() == g["sha256"] and opt == g["opt"]
        out["table_sha256"] = {"match": ok, "sigma": sg, "T": g["T"], "golden": os.path.relpath(gt, ROOT)}
        del t, tv
        torch.cuda.empty_cache()
    if any(v.get("match") is False for v in out.values()):
        print(json.dumps({"parity_failure": out}), flush=True)
        raise SystemExit(3)
    return out


def _config(w, **extra):
    c = {"workload": w.name, "n": w.n, "m": w.m, "eps": w.eps, "P_jobs": w.P, "seed": w.seed,
         "generator": "numpy default_rng(seed).integers(1, P_jobs, n, endpoint=True)"}
    c.update(extra)
    return c


def run_reference(args, w):
    rank, _local, world = _dist_env()
    if rank != 0:
        return 0
    import oracle
    oracle.build()
    N, r, T = _largest_dp(w)
    target = float(os.environ.get("PTAS_REF_SAMPLE_RELAX", "6e8"))
    Nc, _ = _subbox_for(N, r, T, target)
    times, relaxes = [], []
    for i in range(args.warmup + args.steps):
        t0 = time.perf_counter()
        _tab, relax = oracle.dp(Nc, r, T)
        dt = time.perf_counter() - t0
        if i >= args.warmup:
            times.append(dt)
            relaxes.append(relax)
    val = sum(relaxes) / sum(times)
    sample = (f"each step = oracle_dp on the sub-box N'={Nc.tolist()} of the {w.name} DP at T=LB={T} "
              f"({relaxes[0]:.3g} relaxations), sequential C, 1 core")
    line = {"impl": "reference", "metric": METRIC, "value": val, "unit": UNIT, "n_gpus": world,
            "steps": args.steps, "warmup": args.warmup, "ms_per_step": 1e3 * sum(times) / len(times),
            "higher_is_better": True, "scaling": "weak", "vs_baseline": None, "dtype": "int32",
            "data": "synthetic", "config": _config(w, probes_per_round=1, mode="single",
                                                   l2="flushed between steps (256 MiB write)"),
            "cpu_baseline": {"value": val, "unit": UNIT, "cores": 1, "kind": "oracle", "sample": sample},
            "e2e": {"value": val, "unit": UNIT, "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0},
            "gpu_launches": 0}
    print(json.dumps(line), flush=True)
    return 0


def _measure(P, w, opts, lib_stream, flush, local, world, steps, warmup, barrier, clk=None):
    """Warm-up + timed steps of one configuration: device-resident and end-to-end.
    Returns (dev_ms, stats, e2e_ms, e2e_stats)."""
    import torch
    p = w.p()
    n = len(p)
    p_pin = torch.from_numpy(p).pin_memory()
    p_dev = p_pin.to(f"cuda:{local}")
    a_dev = torch.zeros(n, dtype=torch.int32, device=f"cuda:{local}")
    s_ev = torch.cuda.Event(enable_timing=True)
    e_ev = torch.cuda.Event(enable_timing=True)

    def step_device():
        return P.ptas_solve_device(p_dev, w.m, w.eps, a_dev, opts=opts)

    def step_e2e():
        # pinned host p in, host assignment out (the public ABI call a user makes)
        return P.ptas_solve(p_pin.numpy(), w.m, w.eps, opts=opts, log=False)

    def timed(fn, out_ms, out_stats):
        flush.zero_()                       # L2 flush between steps (outside the events)
        torch.cuda.synchronize()
        s_ev.record(lib_stream)
        r = fn()
        e_ev.record(lib_stream)
        torch.cuda.synchronize()
        if out_ms is not None:
            out_ms.append(s_ev.elapsed_time(e_ev))
            out_stats.append(r["stats"])

    dev_ms, stats, e2e_ms, e2e_stats = [], [], [], []
    for _ in range(warmup):        # warm-up steps are identical to the timed ones
        timed(step_device, None, None)
        timed(step_e2e, None, None)
    barrier()
    for _ in range(steps):
        timed(step_device, dev_ms, stats)
    barrier()
    for _ in range(steps):
        timed(step_e2e, e2e_ms, e2e_stats)
    barrier()
    return dev_ms, stats, e2e_ms, e2e_stats


def _reduce(dist, torch, local, world, mode_multi, vals_max, vals_sum):
    """Max over ranks of times, sum over ranks of per-rank work (multi-probe: each
    rank counts only the DPs it ran; level-sharded: every rank counts the same
    DPs, so no sum)."""
    if world == 1:
        return vals_max, vals_sum
    t = torch.tensor(vals_max, dtype=torch.float64, device=f"cuda:{local}")
    dist.all_reduce(t, op=dist.ReduceOp.MAX)
    u = torch.tensor(vals_sum, dtype=torch.float64, device=f"cuda:{local}")
    if mode_multi:
        dist.all_reduce(u, op=dist.ReduceOp.SUM)
    return t.tolist(), u.tolist()


def run_ours(args, w):
    import torch
    import torch.distributed as dist
    import paper_conf_ipps_ligsg18_b200 as P

    rank, local, world = _dist_env()
    torch.cuda.set_device(local)
    if world > 1:
        dist.init_process_group("nccl", device_id=torch.device(f"cuda:{local}"))
    comm = P.init_comm(local) if world > 1 else None
    if world > 1:
        mode = P.MODE_MULTI_PROBE if args.mode == "multiprobe" else P.MODE_LEVEL_SHARDED
        Pp = world if mode == P.MODE_MULTI_PROBE else args.P
    elif args.virtual_shards > 1:
        mode, Pp = P.MODE_LEVEL_SHARDED, args.P
    else:
        mode, Pp = P.MODE_SINGLE, args.P
    # all library work on this stream, so the CUDA events below bracket it exactly
    lib_stream = torch.cuda.Stream(device=local)
    # --slab-pipeline (N > 1, level-sharded): every probe DP windowed and split along
    # the first class over the ranks, halos by ncclSend/ncclRecv
    pipe = args.slab_pipeline and world > 1 and mode == P.MODE_LEVEL_SHARDED
    opts = P.options(P=Pp, mode=mode, device=local, comm=comm, stream=lib_stream,
                     virtual_shards=args.virtual_shards if world == 1 else 1,
                     window=1 if pipe else 0, slab_pipeline=1 if pipe else 0)
    flush = torch.empty(256 << 20, dtype=torch.uint8, device=f"cuda:{local}")

    def barrier():
        if world > 1:
            dist.barrier()
        torch.cuda.synchronize()

    # parity against the oracle's goldens, before anything is timed (rank 0's GPU;
    # the configuration's results do not depend on the rank)
    parity = None
    if not args.no_parity:
        # the solve runs collectively at N > 1 (every rank takes part); rank 0 alone
        # hashes the table
        parity = parity_check(P, w, opts, Pp, table=rank == 0)
        barrier()

    with ClockSampler(local) as clk:
        dev_ms, stats, e2e_ms, e2e_stats = _measure(P, w, opts, lib_stream, flush, local, world, args.steps,
                                                    args.warmup, barrier)
    clocks = clk.summary()
    multi = mode == P.MODE_MULTI_PROBE
    (t_total, e2e_t, fill_s), (relax_total, e2e_relax, alg_bytes, exec_bytes) = _reduce(
        dist, torch, local, world, multi,
        [sum(dev_ms) / 1e3, sum(e2e_ms) / 1e3, sum(s["fill_wall_seconds"] for s in stats)],
        [sum(s["relaxations"] for s in stats), sum(s["relaxations"] for s in e2e_stats),
         sum(s["alg_bytes"] for s in stats), sum(s["exec_bytes"] for s in stats)])
    fill_sum_s = sum(s["fill_seconds"] for s in stats)
    relax_exec = sum(s["relax_executed"] for s in stats)
    fill_launches = sum(s["fill_launches"] for s in stats)
    launches = sum(s["kernel_launches"] for s in stats)
    peak1, peak_kind = _peaks()
    # level-sharded: every rank fills its slice, so the aggregate bandwidth of the
    # job is compared with N GPUs' peak; multi-probe: the ranks' DPs run side by side
    peak = peak1 * world
    # job-wide algorithmic bytes (level-sharded: the one DP every rank fills a slice
    # of; multi-probe: the sum of the ranks' DPs) over the job's fill time (max over ranks)
    achieved = alg_bytes / fill_s / 1e9 if fill_s > 0 else 0.0
    traffic, traffic_note, dram = None, None, None
    tf = os.path.join(ROOT, "profiles", "traffic.json")
    if os.path.exists(tf):
        try:
            t = json.load(open(tf)).get(w.name)
            if t:
                traffic = t["dram_bytes_per_launch"]
                traffic_note = {k: t[k] for k in t if k != "dram_bytes_per_launch"}
                if t.get("dram_gbs"):
                    dram = {"achieved": t["dram_gbs"], "peak": peak1, "unit": "GB/s",
                            "frac": t["dram_gbs"] / peak1, "source": t["source"]}
        except Exception:
            traffic = None
    st0 = stats[0]
    line = {
        "metric": METRIC, "value": relax_total / t_total, "unit": UNIT, "n_gpus": world,
        "steps": args.steps, "warmup": args.warmup, "ms_per_step": 1e3 * t_total / args.steps,
        "higher_is_better": True,
        "scaling": "strong" if (world > 1 and mode == P.MODE_LEVEL_SHARDED) else "weak",
        "vs_baseline": None, "dtype": args.dtype_label or "u8", "data": "synthetic",
        "config": _config(w, probes_per_round=Pp,
                          mode={0: "single", 1: "level_sharded", 2: "multi_probe"}[mode],
                          **({"virtual_shards": args.virtual_shards} if world == 1 and args.virtual_shards > 1 else {}),
                          **({"probe_dps": "windowed, slab/halo pipeline (send/recv)"} if pipe else {}),
                          l2="flushed between steps (256 MiB write)"),
        "solve": {"probes": st0["probes"], "unique_dps": st0["unique_dps"], "T_star": st0["T_star"],
                  "sigma_max": st0["sigma_max"], "K_at_Tstar": st0["K_at_Tstar"],
                  "relax_per_step": relax_total / args.steps,
                  # speculative bisection (D8): DPs evaluated ahead of Alg 1 /
                  # never probed (their work is not in `value`)
                  "spec_dps": st0["spec_dps"], "spec_wasted": st0["spec_wasted"]},
        "solve_ms": 1e3 * t_total / args.steps,
        "solve_ms_median": statistics.median(dev_ms),
        "e2e": {"value": e2e_relax / e2e_t, "unit": UNIT,
                "h2d_bytes_per_step": int(sum(s["h2d_bytes"] for s in e2e_stats) / args.steps),
                "d2h_bytes_per_step": int(sum(s["d2h_bytes"] for s in e2e_stats) / args.steps),
                "solve_ms": 1e3 * e2e_t / args.steps},
        "roofline": {"bound": "hbm", "achieved": achieved, "peak": peak, "unit": "GB/s",
                     "frac": achieved / peak, "traffic": traffic, "traffic_note": traffic_note,
                     "bytes": "SURVEY.md §8(d) algorithmic bytes of Eq. 1: (relaxations + states) * e per DP",
                     "kernel": "level fill (row_fill_swar_kernel dataflow / per-level launches, "
                               "row_ring_kernel for K = 3; §8(a) a-5)",
                     "peak_kind": (peak_kind + " (MEASURED_PEAKS.json hbm_gbs)" if peak_kind == "measured" else "fallback")
                                  + (f" x {world} GPUs" if world > 1 else ""),
                     "fill_ms_per_step": 1e3 * fill_s / args.steps,
                     "fill_time": "union of the DPs' fill intervals (CUDA events, one time axis); "
                                  "alg bytes count only the DPs the search used",
                     "fill_ms_sum_per_step": 1e3 * fill_sum_s / args.steps,
                     "fill_launches_per_step": fill_launches / args.steps,
                     "alg_bytes_per_step": alg_bytes / args.steps,
                     # the kernels take one window per (row, prefix) of the row's pivot block
                     # (D5, D13): the bytes they actually gather, and their rate
                     "relax_executed_per_step": relax_exec / args.steps,
                     "executed_bytes_per_step": exec_bytes / args.steps,
                     "executed_gbs": exec_bytes / fill_s / 1e9 if fill_s > 0 else None,
                     "frac_executed": (exec_bytes / fill_s / 1e9 / peak) if fill_s > 0 else None,
                     "dram": dram,
                     "fill_relax_per_s": relax_total / fill_s if fill_s > 0 else None},
        "parity": parity,
        "step_ms": [round(x, 3) for x in dev_ms],
        "step_dp_ms": [round(1e3 * st["dp_seconds"], 3) for st in stats],
        "step_lib_wall_ms": [round(1e3 * st["total_seconds"], 3) for st in stats],
        "e2e_step_ms": [round(x, 3) for x in e2e_ms],
        "gpu_launches": int(launches),
        "clocks": clocks,
    }
    # secondary blocks (same metric, untimed relative to the line above)
    def block(wb, mode_b, Pb, note):
        ob = P.options(P=Pb, mode=mode_b, device=local, comm=comm if world > 1 else None, stream=lib_stream)
        par = parity_check(P, wb, ob, Pb, table=rank == 0) if not args.no_parity else None
        d, st, e, est = _measure(P, wb, ob, lib_stream, flush, local, world, args.steps, args.warmup, barrier)
        (tt, et), (rr, er) = _reduce(dist, torch, local, world, mode_b == P.MODE_MULTI_PROBE,
                                     [sum(d) / 1e3, sum(e) / 1e3],
                                     [sum(x["relaxations"] for x in st), sum(x["relaxations"] for x in est)])
        return {"workload": wb.name, "mode": {0: "single", 1: "level_sharded", 2: "multi_probe"}[mode_b],
                "probes_per_round": Pb, "n_gpus": world, "value": rr / tt, "unit": UNIT,
                "ms_per_step": 1e3 * tt / args.steps, "e2e_value": er / et, "T_star": st[0]["T_star"],
                "unique_dps": st[0]["unique_dps"], "parity": par, "note": note}
    if not args.no_blocks:
        if world == 1 and w.name != "M4x":
            line["scaling_ref"] = block(WORKLOADS["M4x"], P.MODE_SINGLE, 1,
                                        "north_star's scaling instance on this single GPU: the N = 1 point of the "
                                        "level-sharded 1/2/4/8-GPU curve (bench.py --gpus N defaults to it)")
        if world > 1:
            line["multi_probe"] = block(WORKLOADS["M5s-0.3"], P.MODE_MULTI_PROBE, world,
                                        "multi-section search (Alg 3 generalised, one probe per GPU per round)")
    if rank == 0 and world == 1 and not args.no_cpu_baseline:
        line["cpu_baseline"] = cpu_oracle_sample(w)
    if comm is not None:
        comm.destroy()
    if rank == 0:
        print(json.dumps(line), flush=True)
    if world > 1:
        dist.destroy_process_group()
    return 0


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=20)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--impl", choices=["ours", "reference"], default="ours")
    ap.add_argument("--workload", default=None, choices=sorted(WORKLOADS),
                    help="default: M2s at N = 1, M4x (level-sharded) at N > 1")
    ap.add_argument("--P", type=int, default=1, help="probes per round (single GPU)")
    ap.add_argument("--mode", choices=["auto", "sharded", "multiprobe"], default="auto",
                    help="N>1 mode; auto = sharded when the workload's largest table is >= 1 GB "
                         "(M3g, M4x), else multiprobe (DESIGN.md §9: level sharding only pays on large tables)")
    ap.add_argument("--virtual-shards", type=int, default=1,
                    help="N=1 only: run LEVEL_SHARDED with G logical shards on one GPU (slice fill + "
                         "gather copy + scatter per level, no NCCL) to measure the exchange overhead")
    ap.add_argument("--slab-pipeline", action="store_true",
                    help="N > 1 level-sharded: windowed probe DPs on the slab/halo pipeline (send/recv)")
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--no-parity", action="store_true", help="skip the oracle-golden parity assertion")
    ap.add_argument("--no-blocks", action="store_true", help="skip the scaling_ref / multi_probe blocks")
    ap.add_argument("--dtype-label", default=None)
    args = ap.parse_args()
    _rank, _local, world = _dist_env()
    if args.workload is None:
        args.workload = "M2s" if world == 1 else "M4x"
    w = WORKLOADS[args.workload]
    # geometry of the largest DP: the product's host ABI for our arm, the
    # oracle only on the reference (oracle) arm
    N, _r, _T = _largest_dp(w) if args.impl == "reference" else _largest_dp_product(w)
    e = 1 if int(np.sum(N)) <= 255 else 2
    if args.dtype_label is None:
        args.dtype_label = "u8" if e == 1 else "u16"
    if args.mode == "auto":
        table_bytes = float(np.prod(np.asarray(N, np.float64) + 1)) * e if len(N) else 0.0
        args.mode = "sharded" if table_bytes >= 1e9 else "multiprobe"
    if args.impl == "reference":
        return run_reference(args, w)
    return run_ours(args, w)


if __name__ == "__main__":
    sys.exit(main())

"""D* direct dp_fill roofline sweep: no search, one DP per
(k, K, sigma_target) from synth.dstar, filled by dp_fill_device into a
caller-owned torch buffer; CUDA events on the library stream around the call.

relax = closed form sum_{s in C} prod(N_i - s_i + 1) (C from dp_configs);
roofline = relax * e bytes / time against MEASURED_PEAKS.json hbm_gbs.
Prints one JSON line per DP.  Run under gpurun (1 GPU)."""
from __future__ import annotations

import json
import os
import sys

import numpy as np
import torch

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import paper_conf_ipps_ligsg18_b200 as P  # noqa: E402
from synth import dstar  # noqa: E402

peak = json.load(open(os.path.join(ROOT, "MEASURED_PEAKS.json")))["hbm_gbs"]
targets = [float(x) for x in os.environ.get("DSWEEP_SIGMA", "1e6,1e7,1e8,1e9,4e9").split(",")]
reps = int(os.environ.get("DSWEEP_REPS", "3"))
Ks = [int(x) for x in os.environ.get("DSWEEP_K", "3,4,5,6,7,8").split(",")]
torch.cuda.set_device(0)
stream = torch.cuda.Stream()
flush = torch.empty(256 << 20, dtype=torch.uint8, device="cuda")
for k in (4, 5, 7):
    for K in Ks:
        for st in targets:
            N, r, T = dstar(K, st, k)
            sigma, e = P.dp_table_shape(N)
            C = P.dp_configs(N, r, T)
            relax = float(sum(np.prod((N - s + 1).astype(np.float64)) for s in C))
            if relax > 2.0e13:
                continue
            tab = torch.empty(sigma * e, dtype=torch.uint8, device="cuda")
            times = []
            with torch.cuda.stream(stream):
                for i in range(reps + 1):
                    flush.fill_(i)
                    a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
                    torch.cuda.synchronize()
                    a.record(stream)
                    opt = P.dp_fill_device(N, r, T, tab, stream)
                    b.record(stream)
                    torch.cuda.synchronize()
                    if i:
                        times.append(a.elapsed_time(b) / 1e3)
            t = min(times)
            gbs = relax * e / t / 1e9
            print(json.dumps({"k": k, "K": K, "sigma_target": st, "N": N.tolist(), "T": T, "sigma": sigma,
                              "e": e, "C": len(C), "relax": relax, "opt_N": opt, "dp_ms": 1e3 * t,
                              "relax_per_s": relax / t, "gather_gbs": gbs, "frac": gbs / peak}), flush=True)
            del tab
            torch.cuda.empty_cache()

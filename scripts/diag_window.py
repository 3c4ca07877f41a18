"""Device time of the workload's largest DP with and without the level window
(dp_fill_opt), median of R: python scripts/diag_window.py W [R] [budget_bytes]"""
import os, sys, statistics, time
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import paper_conf_ipps_ligsg18_b200 as P
from synth import WORKLOADS
torch.cuda.set_device(0)
name = sys.argv[1]
R = int(sys.argv[2]) if len(sys.argv) > 2 else 5
w = WORKLOADS[name]
p = w.p()
k = P.ptas_k(w.eps)
LB, _ = P.ptas_bounds(p, w.m)
u, r, N, _ = P.ptas_classify(p, LB, k)
for win in (-1, 1):
    ms, st = [], None
    for i in range(R + 1):
        opt, st = P.dp_fill_opt(N, r, LB, window=win)
        if i:
            ms.append(1e3 * st["fill_seconds"])
    print(f"{name} window={win} opt={opt} fill_ms={statistics.median(ms):.3f} dev_bytes={st['dev_bytes_max'] / 1e6:.1f} MB "
          f"windowed={st['window_dps']}", flush=True)

"""Device time of the workload's largest DP (T = LB, solve layout) through
dp_fill_device, median of R runs: python scripts/diag_dp.py W [R]
(env knobs of the engine apply; used for A/B runs under gpurun)."""
import os, sys, statistics
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
import torch
import paper_conf_ipps_ligsg18_b200 as P
from synth import WORKLOADS
torch.cuda.set_device(0)
name = sys.argv[1]
R = int(sys.argv[2]) if len(sys.argv) > 2 else 10
w = WORKLOADS[name]
p = w.p()
k = P.ptas_k(w.eps)
LB, _ = P.ptas_bounds(p, w.m)
u, r, N, _ = P.ptas_classify(p, LB, k)
o = P.ptas_table_order(N, r, 0)
N, r = N[o], r[o]
sg, e = P.dp_table_shape(N)
t = torch.empty(sg * e, dtype=torch.uint8, device="cuda")
s = torch.cuda.current_stream()
a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
ms = []
for i in range(R + 2):
    a.record(s)
    opt = P.dp_fill_device(N, r, LB, t)
    b.record(s)
    torch.cuda.synchronize()
    if i >= 2:
        ms.append(a.elapsed_time(b))
lv = int(N[:-1].sum()) + 1
print(f"{name} N={N.tolist()} sigma={sg:.3g} levels={lv} opt={opt} dp_ms={statistics.median(ms):.3f} "
      f"us/level={1e3 * statistics.median(ms) / lv:.2f} env={ {k: v for k, v in os.environ.items() if k.startswith('PTAS_')} }", flush=True)

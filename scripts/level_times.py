"""Largest DP (T = LB) of a workload in the solve's internal class order through
dp_fill, alone on the GPU; PTAS_LEVEL_TIMES=1 prints the per-row-level device
times (us) and row counts.  Usage: PTAS_LEVEL_TIMES=1 python scripts/level_times.py M2s"""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
import paper_conf_ipps_ligsg18_b200 as P
from synth import WORKLOADS

w = WORKLOADS[sys.argv[1] if len(sys.argv) > 1 else "M2s"]
p = w.p()
k = P.ptas_k(w.eps)
LB, UB = P.ptas_bounds(p, w.m)
u, r, N, _ = P.ptas_classify(p, LB, k)
o = P.ptas_table_order(N, r)
N, r = N[o].astype(np.int32), r[o].astype(np.int64)
for i in range(int(sys.argv[2]) if len(sys.argv) > 2 else 3):
    opt, _, st = P.dp_fill(N, r, LB, table=False)
    print("rep %d fill %.3f ms launches %d" % (i, 1e3 * st["fill_seconds"], st["fill_launches"]), flush=True)

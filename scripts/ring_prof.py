"""Largest DP (T = LB) of a K = 3 workload through dp_fill, timed (CUDA events around
the call); with a -DPTAS_RING_PROFILE=1 variant library the ring kernel prints
its per-level cycle breakdown.  Usage: python scripts/ring_prof.py M5s-0.3 [reps]"""
import os, sys, time
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
import paper_conf_ipps_ligsg18_b200 as P
from synth import WORKLOADS

w = WORKLOADS[sys.argv[1] if len(sys.argv) > 1 else "M5s-0.3"]
reps = int(sys.argv[2]) if len(sys.argv) > 2 else 5
p = w.p()
k = P.ptas_k(w.eps)
LB, UB = P.ptas_bounds(p, w.m)
u, r, N, _ = P.ptas_classify(p, LB, k)
o = P.ptas_table_order(N, r)            # the solve's internal class order
N, r = N[o].astype(np.int32), r[o].astype(np.int64)
print(w.name, "LB", LB, "N", N.tolist(), "r", r.tolist(), flush=True)
for i in range(reps):
    t0 = time.perf_counter()
    opt, tab, st = P.dp_fill(N, r, LB)
    t1 = time.perf_counter()
    print("rep %d opt %d wall %.3f ms fill %.3f ms" % (i, opt, 1e3 * (t1 - t0), 1e3 * st.get("fill_seconds", 0.0)), flush=True)

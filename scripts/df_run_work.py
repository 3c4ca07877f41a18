"""Relaxations and rows of the dataflow warp-mode run of a workload's T = LB DP
(the levels with more than PTAS_DF_SPLIT_ROWS rows): the longest fill launch
of a solve, for make_profiles.py (closed form, scripts/level_work.py)."""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
sys.path.insert(0, os.path.dirname(os.path.abspath(__file__)))
import numpy as np
import oracle
from synth import WORKLOADS
from level_work import level_relax

w = WORKLOADS[sys.argv[1]]
thr = int(os.environ.get("PTAS_DF_SPLIT_ROWS", "2000"))
p = w.p(); k = oracle.k_of(w.eps); LB, _ = oracle.bounds(p, w.m)
u, r, N, _ = oracle.classify(p, LB, k)
rows, rel, W, nC = level_relax(N, r, LB)
sel = rows > thr
print(f"{rel[sel].sum():.6g} {rows[sel].sum():.6g} {W}")

"""A/B timing of library variants: median solve / fill time over repeated solves
(PTAS_LIB selects the variant; PTAS_SPEC_DEPTH=0 for clean per-DP fill sums)."""
import os, statistics, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import paper_conf_ipps_ligsg18_b200 as P
from synth import WORKLOADS
torch.cuda.set_device(0)
tag = os.environ.get("TAG", os.environ.get("PTAS_LIB", "base") or "base")
for name in sys.argv[1:]:
    w = WORKLOADS[name]
    p = w.p()
    tot, fill = [], []
    for i in range(int(os.environ.get("REPS", "8"))):
        r = P.ptas_solve(p, w.m, w.eps, P=1, log=False)
        if i >= 2:
            tot.append(r["stats"]["total_seconds"] * 1e3)
            fill.append(r["stats"]["fill_seconds"] * 1e3)
    print(f"{tag:40s} {name:9s} total {statistics.median(tot):8.3f} ms  fill {statistics.median(fill):8.3f} ms  relax {r['stats']['relaxations']:.3g}", flush=True)

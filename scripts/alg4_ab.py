"""A/B of the paper's Alg 4 data partitioning (dp_fill_alg4, csrc/alg4.cu) against
this engine's level fill (dp_fill_opt, full table) on the largest DP of each
workload: device fill time (CUDA events), same OPT.  python scripts/alg4_ab.py W..."""
import os, sys, statistics, time
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import paper_conf_ipps_ligsg18_b200 as P
from synth import WORKLOADS
torch.cuda.set_device(0)
for name in sys.argv[1:]:
    w = WORKLOADS[name]
    p = w.p()
    k = P.ptas_k(w.eps)
    LB, _ = P.ptas_bounds(p, w.m)
    u, r, N, _ = P.ptas_classify(p, LB, k)
    ours = []
    for i in range(4):
        opt, st = P.dp_fill_opt(N, r, LB, window=-1)
        if i:
            ours.append(1e3 * st["fill_seconds"])
    line = f"{name} K={len(N)} sigma={st['states']:.3g} relax={st['relaxations']:.3g} ours fill {statistics.median(ours):.3f} ms (opt {opt})"
    for dim in (3, 6, 9):
        t0 = time.time()
        o4, _t, div, s4 = P.dp_fill_alg4(N, r, LB, dim=dim, table=False)
        assert o4 == opt
        line += f" | alg4 dim={dim} div={div} {1e3 * s4['fill_seconds']:.1f} ms ({s4['fill_launches']} block-levels, x{s4['fill_seconds'] * 1e3 / statistics.median(ours):.0f})"
        if time.time() - t0 > 60:
            break
    print(line, flush=True)

"""Per-DP trace of one solve (PTAS_TRACE=1 prints per DP lines on stderr)."""
import os, sys, time
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import paper_conf_ipps_ligsg18_b200 as P
from synth import WORKLOADS
torch.cuda.set_device(0)
for name in sys.argv[1:]:
    w = WORKLOADS[name]
    p = w.p()
    for i in range(3):
        r = P.ptas_solve(p, w.m, w.eps, P=int(os.environ.get("PP", "1")), log=True)
    s = r["stats"]
    print(f"== {name} T*={r['T_star']} total={1e3*s['total_seconds']:.2f} ms fill={1e3*s['fill_seconds']:.2f} dps={s['unique_dps']} probes={s['probes']}", flush=True)
    for pr in r["probes"]:
        print("  probe T=%d round=%d feas=%d K=%d opt=%d sigma=%d memo=%d" % pr, flush=True)

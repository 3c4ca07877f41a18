import os, sys, time
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import paper_conf_ipps_ligsg18_b200 as P
from synth import WORKLOADS
w = WORKLOADS[os.environ.get("WL", "M2s")]
torch.cuda.set_device(0)
p = w.p()
for budget in (0, 64 << 30):
    for i in range(4):
        t0 = time.perf_counter()
        r = P.ptas_solve(p, w.m, w.eps, P=1, log=False, budget=budget)
        t1 = time.perf_counter()
        s = r["stats"]
        print(f"budget={budget>>30}G wall={1e3*(t1-t0):7.2f} ms total={1e3*s['total_seconds']:7.2f} dp={1e3*s['dp_seconds']:7.2f} fill={1e3*s['fill_seconds']:7.2f} launches={s['kernel_launches']}")

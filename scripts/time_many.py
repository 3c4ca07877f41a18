"""Repeated solves: host wall vs device DP time per solve (host-overhead diagnostics)."""
import os, sys, time
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import paper_conf_ipps_ligsg18_b200 as P
from synth import WORKLOADS
torch.cuda.set_device(0)
w = WORKLOADS[sys.argv[1]]
p = w.p()
for i in range(int(sys.argv[2]) if len(sys.argv) > 2 else 10):
    t0 = time.perf_counter()
    r = P.ptas_solve(p, w.m, w.eps, P=int(os.environ.get("PP", "1")), log=False)
    t1 = time.perf_counter()
    s = r["stats"]
    print(f"wall={1e3*(t1-t0):8.2f} total={1e3*s['total_seconds']:8.2f} dp={1e3*s['dp_seconds']:8.2f} fill={1e3*s['fill_seconds']:8.2f} dps={s['unique_dps']}", flush=True)
if os.environ.get("WITH_STREAM"):
    st = torch.cuda.Stream()
    o = P.options(P=1, stream=st, device=0)
    for i in range(8):
        t0 = time.perf_counter()
        r = P.ptas_solve(p, w.m, w.eps, opts=o, log=False)
        t1 = time.perf_counter()
        s = r["stats"]
        print(f"[stream] wall={1e3*(t1-t0):8.2f} total={1e3*s['total_seconds']:8.2f} dp={1e3*s['dp_seconds']:8.2f} fill={1e3*s['fill_seconds']:8.2f}", flush=True)
    pd = torch.from_numpy(p).cuda(); a = torch.zeros(len(p), dtype=torch.int32, device="cuda")
    for i in range(8):
        t0 = time.perf_counter()
        r = P.ptas_solve_device(pd, w.m, w.eps, a, opts=o)
        t1 = time.perf_counter()
        s = r["stats"]
        print(f"[device] wall={1e3*(t1-t0):8.2f} total={1e3*s['total_seconds']:8.2f} dp={1e3*s['dp_seconds']:8.2f} fill={1e3*s['fill_seconds']:8.2f}", flush=True)

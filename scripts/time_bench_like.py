import os, sys, time
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import paper_conf_ipps_ligsg18_b200 as P
from synth import WORKLOADS
w = WORKLOADS["M2s"]
torch.cuda.set_device(0)
p = w.p()
p_pin = torch.from_numpy(p).pin_memory()
p_dev = p_pin.to("cuda:0")
a_dev = torch.zeros(len(p), dtype=torch.int32, device="cuda:0")
flush = torch.empty(256 << 20, dtype=torch.uint8, device="cuda:0")
opts = P.options(P=1, mode=P.MODE_SINGLE, device=0)
s_ev = torch.cuda.Event(enable_timing=True); e_ev = torch.cuda.Event(enable_timing=True)
for variant in ("dev", "host", "dev_noflush", "host_np"):
    for i in range(5):
        if "noflush" not in variant:
            flush.zero_()
        torch.cuda.synchronize()
        s_ev.record(); t0 = time.perf_counter()
        if variant.startswith("dev"):
            r = P.ptas_solve_device(p_dev, w.m, w.eps, a_dev, opts=opts)
        elif variant == "host":
            r = P.ptas_solve(p_pin.numpy(), w.m, w.eps, opts=opts, log=False)
        else:
            r = P.ptas_solve(p, w.m, w.eps, opts=opts, log=False)
        t1 = time.perf_counter(); e_ev.record(); torch.cuda.synchronize()
        s = r["stats"]
        print(f"{variant:12s} ev={s_ev.elapsed_time(e_ev):7.2f} wall={1e3*(t1-t0):7.2f} total={1e3*s['total_seconds']:7.2f} dp={1e3*s['dp_seconds']:7.2f}")

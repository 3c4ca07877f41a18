import os, sys, time, threading
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import paper_conf_ipps_ligsg18_b200 as P
from synth import WORKLOADS
w = WORKLOADS[os.environ.get("WL", "M2s")]
torch.cuda.set_device(0)
p = w.p()
flush = torch.empty(256 << 20, dtype=torch.uint8, device="cuda:0")
def run(tag, pre=None, n=4):
    for i in range(n):
        if pre: pre()
        torch.cuda.synchronize()
        t0 = time.perf_counter()
        r = P.ptas_solve(p, w.m, w.eps, P=1, log=False)
        t1 = time.perf_counter()
        s = r["stats"]
        print(f"{tag:12s} wall={1e3*(t1-t0):7.2f} dp={1e3*s['dp_seconds']:7.2f} fill={1e3*s['fill_seconds']:7.2f}")
run("plain")
run("flush", lambda: flush.zero_())
run("fill255", lambda: flush.fill_(255))
stop = threading.Event()
def samp():
    import pynvml as nv
    nv.nvmlInit(); h = nv.nvmlDeviceGetHandleByIndex(0)
    while not stop.is_set():
        nv.nvmlDeviceGetClockInfo(h, nv.NVML_CLOCK_SM); nv.nvmlDeviceGetCurrentClocksEventReasons(h); stop.wait(0.1)
th = threading.Thread(target=samp, daemon=True); th.start()
run("nvml")
run("nvml+flush", lambda: flush.zero_())
stop.set()

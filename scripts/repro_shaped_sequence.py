"""Runs the shaped-workload golden solves in the test order (M2s, M3s, M5s-*, P = 1/2/4/8) N times in one
process and reports probe-log mismatches against the oracle goldens (regression check for the
round-trip-free enumeration race, D9).  Usage: python scripts/repro_shaped_sequence.py [N]"""
import json, os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import paper_conf_ipps_ligsg18_b200 as P
from synth import WORKLOADS
gold = {}
for name in ["M2s", "M3s", "M5s-0.15", "M5s-0.2", "M5s-0.3"]:
    for Pp in [1, 2, 4, 8]:
        f = f"tests/golden/shaped/solve_{name}_P{Pp}.json"
        if os.path.exists(f): gold[(name, Pp)] = json.load(open(f))
bad = 0
for it in range(int(sys.argv[1]) if len(sys.argv) > 1 else 6):
    for (name, Pp), g in gold.items():
        w = WORKLOADS[name]
        got = P.ptas_solve(w.p(), w.m, w.eps, P=Pp)
        gp = [list(x[:6]) for x in got["probes"]]
        wp = [list(x) for x in g["probes"]]
        d = [(i, a, b) for i, (a, b) in enumerate(zip(gp, wp)) if a != b]
        if d:
            bad += 1
            print(it, name, Pp, d[:2], flush=True)
print("bad", bad, flush=True)

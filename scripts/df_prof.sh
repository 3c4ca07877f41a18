#!/bin/bash
# per-level DF timelines (diagnostics build variants/prof)
cat > /tmp/one.py <<'PY'
import os, sys
sys.path.insert(0, os.getcwd())
import paper_conf_ipps_ligsg18_b200 as P
from synth import WORKLOADS
w = WORKLOADS[os.environ.get("WL", "M2s")]
for i in range(2):
    r = P.ptas_solve(w.p(), w.m, w.eps, P=1, log=False)
print("fill ms", r["stats"]["fill_seconds"] * 1e3)
PY
for W in ${WLS:-M2s}; do
 for M in ${MODES:-3}; do
  PTAS_LIB=variants/prof/libptas_b200.so PTAS_DF=$M PTAS_DF_SPLIT_ROWS=${SPLIT:-2000} PTAS_DF_PROF=1 WL=$W PTAS_TRACE=1 python /tmp/one.py > gpurun_out/dfprof_${W}_$M.log 2>&1
 done
done

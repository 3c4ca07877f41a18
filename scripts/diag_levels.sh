#!/bin/bash
# per-level device times + host trace + slow calls (run under gpurun)
mkdir -p gpurun_out
for W in ${WLS:-M2s M3s M5s-0.3 M4x}; do
  WL=$W PTAS_LEVEL_TIMES=1 timeout 300 python scripts/time_solve.py > gpurun_out/lev_$W.log 2>&1
  WL=$W PTAS_TRACE=1 PTAS_SLOW_CALLS=3 timeout 300 python scripts/time_solve.py > gpurun_out/trace_$W.log 2>&1
done

#!/bin/bash
# A/B of the fill modes on the solve workloads (run under gpurun)
mkdir -p gpurun_out
for W in ${WLS:-M2s M3s M5s-0.3 M5s-0.15 M4s}; do
  for M in ${MODES:-0 1 2}; do
    echo "== $W PTAS_DF=$M $EXTRA"
    WL=$W PTAS_DF=$M timeout 300 python scripts/time_solve.py 2>&1 | tail -2
  done
done

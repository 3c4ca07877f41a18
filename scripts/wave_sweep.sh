#!/bin/bash
for W in ${WLS:-M2s M3s M5s-0.3 M5s-0.15 M4s}; do
 for WV in ${WAVES:-1 2 4 1000}; do
  for D in ${DEPTHS:-0 3}; do
    echo "== $W wave=$WV spec=$D"; WL=$W PTAS_DF_WAVE=$WV PTAS_SPEC_DEPTH=$D timeout 300 python scripts/time_solve.py 2>&1 | tail -1
  done
 done
done

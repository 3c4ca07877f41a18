#!/bin/bash
for W in ${WLS:-M2s M3s M5s-0.3 M5s-0.15 M4s}; do
  for D in ${DEPTHS:-0 1 2 3}; do
    echo "== $W spec_depth=$D sigma=${PTAS_SPEC_SIGMA:-default}"; WL=$W PTAS_SPEC_DEPTH=$D timeout 300 python scripts/time_solve.py 2>&1 | tail -1
  done
done

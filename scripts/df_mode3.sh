#!/bin/bash
for W in ${WLS:-M2s M3s M5s-0.3 M5s-0.15 M4s}; do
  for S in ${SPLITS:-0 600 2000 8000 30000}; do
    echo "== $W DF=3 split_rows=$S"; WL=$W PTAS_DF=3 PTAS_DF_SPLIT_ROWS=$S timeout 300 python scripts/time_solve.py 2>&1 | tail -1
  done
done

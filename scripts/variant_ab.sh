#!/bin/bash
# A/B of library variants (variants/<name>/libptas_b200.so; "base" = in-tree) on solve workloads
for V in ${VARS:-base}; do
  if [ $V = base ]; then L=""; else L=variants/$V/libptas_b200.so; fi
  for W in ${WLS:-M2s M4s}; do
    echo "== $V $W $EXTRA"; PTAS_LIB=$L WL=$W timeout 300 python scripts/time_solve.py 2>&1 | tail -1
  done
done

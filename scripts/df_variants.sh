#!/bin/bash
# A/B of compile-time variants in DF mode (run under gpurun)
for V in base pb2x8 cg; do
  if [ $V = base ]; then L=""; else L=variants/$V/libptas_b200.so; fi
  for W in M2s M3s M4s M5s-0.3; do
    echo "== $V $W DF=1"; PTAS_LIB=$L WL=$W PTAS_DF=1 timeout 300 python scripts/time_solve.py 2>&1 | tail -1
  done
  echo "== $V M2s DF=1 CH=1"; PTAS_LIB=$L WL=M2s PTAS_DF=1 PTAS_DF_CH=1 timeout 300 python scripts/time_solve.py 2>&1 | tail -1
done

#!/bin/bash
# A/B over library variants x env settings (run under gpurun); VARS, WLS, ENVS
for V in ${VARS:-base}; do
  if [ $V = base ]; then L=""; else L=variants/$V/libptas_b200.so; fi
  for E in ${ENVS:-none}; do
    if [ $E = none ]; then EV=""; else EV="${E//,/ }"; fi
    env $EV PTAS_LIB=$L TAG="$V $E" timeout 300 python scripts/ab_fill.py ${WLS:-M2s M4s} 2>&1 | grep -v Warning
  done
done

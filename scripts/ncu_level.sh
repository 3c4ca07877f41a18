#!/bin/bash
# --set full on the N-th row_fill launch of one solve: scripts/ncu_level.sh <WL> <skip> <tag>
export WL=$1
ncu --set full --clock-control none --import-source on -k regex:row_fill -s $2 -c 1 -o gpurun_out/$3 python scripts/profile_solve.py > /dev/null 2>&1

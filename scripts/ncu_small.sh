#!/bin/bash
# --set full on a small row-level launch (level 3 of the first DP of one solve)
export WL=${1:-M2s}
ncu --set full --clock-control none --import-source on -k regex:row_fill -s 3 -c 1 -o gpurun_out/${2:-small}_full python scripts/profile_solve.py > /dev/null 2>&1

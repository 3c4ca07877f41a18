#!/bin/bash
# usage: scripts/ncu_top.sh <tag> [workload]   (run under gpurun; 1 GPU)
# 1) launch list of one solve  2) --set full on the longest row_fill launch
set -e
TAG=$1; WL=${2:-M2s}
export WL
ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/${TAG}_launches.csv \
    python scripts/profile_solve.py > /dev/null 2>&1
IDX=$(python - <<PY
import csv
rows=[r for r in csv.DictReader(l for l in open("gpurun_out/${TAG}_launches.csv") if not l.startswith("=="))]
fill=[r for r in rows if "row_fill" in r["Kernel Name"]]
best=max(range(len(fill)), key=lambda i: float(fill[i]["Metric Value"].replace(",","")))
print(best)
PY
)
echo "longest row_fill launch ordinal: $IDX"
ncu --set full --clock-control none --import-source on -k regex:row_fill -s $IDX -c 1 \
    -o gpurun_out/${TAG}_full python scripts/profile_solve.py > /dev/null 2>&1
ls -la gpurun_out/

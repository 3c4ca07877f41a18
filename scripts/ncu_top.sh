#!/bin/bash
# usage: scripts/ncu_top.sh <tag> [workload]   (run under gpurun; 1 GPU)
# 1) launch list of one solve (gpu__time_duration per launch, clocks not locked)
# 2) launch list of the workload's largest DP alone (scripts/diag_dp.py: single
#    thread, deterministic launch order) and ncu --set full (+ DRAM throughput /
#    L2 hit metrics) on its longest level-fill launch
set -e
TAG=$1; WL=${2:-M2s}
export WL
ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/${TAG}_launches.csv \
    python scripts/profile_solve.py > /dev/null 2>&1
ncu --metrics gpu__time_duration.sum --clock-control none --csv -k regex:'row_fill|row_ring' \
    --log-file gpurun_out/${TAG}_dplaunches.csv python scripts/diag_dp.py $WL 1 > /dev/null 2>&1
IDX=$(python - <<PY
import csv
rows=[r for r in csv.DictReader(l for l in open("gpurun_out/${TAG}_dplaunches.csv") if not l.startswith("=="))]
best=max(range(len(rows)), key=lambda i: float(rows[i]["Metric Value"].replace(",","")))
print(best)
PY
)
echo "longest level-fill launch ordinal: $IDX"
ncu --set full --metrics dram__bytes.sum.per_second,dram__throughput.avg.pct_of_peak_sustained_elapsed,lts__t_sector_hit_rate.pct \
    --clock-control none --import-source on -k regex:'row_fill|row_ring' -s $IDX -c 1 \
    -o gpurun_out/${TAG}_full python scripts/diag_dp.py $WL 1 > /dev/null 2>&1

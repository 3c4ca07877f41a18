# End-of-round ncu evidence (under gpurun, 1 GPU): the launch list of the bench
# command, --set full of the longest level-fill launch of M2s and M5s-0.3, and
# the bench line itself (run first, without ncu).  TAG=<prefix> (default r02f).
TAG=${TAG:-r02f}
mkdir -p gpurun_out
python bench.py > gpurun_out/${TAG}_bench.log 2>&1 && tail -1 gpurun_out/${TAG}_bench.log > gpurun_out/${TAG}_bench.json
ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/${TAG}_bench_launches.csv \
    python bench.py --steps 2 --warmup 1 --no-cpu-baseline --no-blocks --no-parity > gpurun_out/${TAG}_bench_ncu.log 2>&1
python scripts/ncu_launches.py gpurun_out/${TAG}_bench_launches.csv \
    "${TAG}: launch list of \`python bench.py --steps 2 --warmup 1 --no-cpu-baseline --no-blocks --no-parity\` (M2s)" > gpurun_out/${TAG}_bench_launches.md
for W in ${WLS:-M2s M5s-0.3}; do
  bash scripts/ncu_top.sh ${TAG}_$W $W && python scripts/ncu_summarize.py ${TAG}_$W $W
done
ls gpurun_out/${TAG}*

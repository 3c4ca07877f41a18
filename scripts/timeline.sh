# host timeline of one solve per workload (PTAS_TRACE=1; scripts/timeline.py)
for W in ${WLS:-M5s-0.3 M2s}; do PTAS_TRACE=1 python scripts/trace_solve.py $W > gpurun_out/tl_$W.log 2>&1; echo "== $W"; python scripts/timeline.py gpurun_out/tl_$W.log; done

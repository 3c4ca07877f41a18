# ring-kernel per-level breakdown (variant build with -DPTAS_RING_PROFILE=1) + solve traces
mkdir -p gpurun_out
[ -f variants/ringprof/libptas_b200.so ] || PTAS_VARIANT=ringprof PTAS_EXTRA_FLAGS="-DPTAS_RING_PROFILE=1" python paper_conf_ipps_ligsg18_b200/build.py > gpurun_out/rp_build.log 2>&1 || exit 1
for W in M5s-0.3 M5s-0.2; do
  PTAS_LIB=variants/ringprof/libptas_b200.so python scripts/ring_prof.py $W 3 > gpurun_out/rp_$W.log 2>&1
  python scripts/ring_prof.py $W 5 >> gpurun_out/rp_$W.log 2>&1
done
for W in M5s-0.3 M2s; do PTAS_TRACE=1 python scripts/trace_solve.py $W > gpurun_out/tr_$W.log 2>&1; done
tail -n 30 gpurun_out/rp_*.log gpurun_out/tr_*.log

# A/B of environment knobs on bench.py solves: WLS="M2s M4s" ENVS="X=1 Y=2,Z=3" (comma = several vars)
mkdir -p gpurun_out
for W in ${WLS:-M2s}; do
  for E in ${ENVS:-NONE=0}; do
    env ${E//,/ } timeout 300 python bench.py --workload $W --no-cpu-baseline --no-blocks --steps ${STEPS:-10} --warmup 3 > gpurun_out/kab_${W}_${E//[,=\/]/_}.log 2>&1
    tail -1 gpurun_out/kab_${W}_${E//[,=\/]/_}.log | python -c "
import json,sys
try:
  d=json.loads(sys.stdin.read()); r=d['roofline']
  print('$W $E solve %.3f ms (med %.3f) fill %.3f ms frac %.3f parity %s/%s' % (d['ms_per_step'], d['solve_ms_median'], r['fill_ms_per_step'], r['frac'], d['parity']['solve']['match'], d['parity']['table_sha256']['match']))
except Exception as e: print('$W $E failed', e)"
  done
done

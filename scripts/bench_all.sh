#!/bin/bash
# bench.py over the workload table (run under gpurun); one JSON line per workload
mkdir -p gpurun_out
for W in ${WLS:-M2s M3s M3g M4s M4x M5s-0.3 M5s-0.2 M5s-0.15}; do
  timeout 600 python bench.py --workload $W --no-cpu-baseline --steps ${STEPS:-5} --warmup 3 > gpurun_out/ball_$W.log 2>&1
  tail -1 gpurun_out/ball_$W.log | python -c "
import json,sys
try:
  d=json.loads(sys.stdin.read()); r=d['roofline']
  print('$W', 'solve %.2f ms'%d['ms_per_step'], 'fill %.2f ms'%r['fill_ms_per_step'], 'relax/s %.3g'%d['value'], 'fill relax/s %.3g'%r['fill_relax_per_s'], 'frac %.3f'%r['frac'], 'exec/eq1 %.2f'%(r['relax_executed_per_step']/d['solve']['relax_per_step']), 'K', d['solve'].get('K_at_Tstar'), 'sigma %.3g'%d['solve']['sigma_max'], 'spec', d['solve'].get('spec_dps'), d['solve'].get('spec_wasted'))
except Exception as e: print('$W failed', e)
"
done

PTAS_TRACE=1 python scripts/trace_solve.py M5s-0.2 > gpurun_out/ab2_tr.log 2>&1; grep ring gpurun_out/ab2_tr.log | sort | uniq -c | head; tail -12 gpurun_out/ab2_tr.log
WLS="M5s-0.3 M5s-0.2" ENVS="NONE=0 PTAS_RING_CS=8 PTAS_RING_CS=8,PTAS_RING_P2P=1" bash scripts/knob_ab.sh

timeout 900 python -m pytest tests/test_gpu_ring.py -m gpu -q -x 2>&1 | tail -2
PTAS_TRACE=1 python scripts/trace_solve.py M5s-0.2 > gpurun_out/ab3_tr.log 2>&1; grep ring gpurun_out/ab3_tr.log | sort | uniq -c | head
WLS="M5s-0.3 M5s-0.2" ENVS="NONE=0 PTAS_RING_P2P=1 PTAS_RING_P2P=1,PTAS_RING_EXTRA=0" bash scripts/knob_ab.sh
WLS="M2s M4s M3s" ENVS="NONE=0 PTAS_GRID_SHARE=1" bash scripts/knob_ab.sh

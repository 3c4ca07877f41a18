timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_shaped.py -m gpu -q -x -k "traceback or solve or shaped or hmbp" 2>&1 | tail -2
bash scripts/r02_tl.sh 2>&1 | grep -E "==|traceback|solve"
WLS="M5s-0.3 M5s-0.2 M2s" ENVS="NONE=0 PTAS_TB_REG=0" bash scripts/knob_ab.sh
WLS="M2s M4s M4x M3g" ENVS="NONE=0 PTAS_LIB=variants/minb4/libptas_b200.so" bash scripts/knob_ab.sh

#!/bin/bash
# quick GPU loop: parity subset + bench (run under gpurun)
set -o pipefail
timeout 900 python -m pytest tests/test_gpu_parity.py -x -q ${PYTEST_K:+-k "$PYTEST_K"} 2>&1 | tail -15
timeout 600 python bench.py --steps 3 --warmup 2 --no-cpu-baseline ${BENCH_ARGS} 2>&1 | tail -3

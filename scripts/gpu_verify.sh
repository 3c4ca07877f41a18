set -x
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv
python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/v1_smoke.log 2>&1; echo smoke rc=$?
timeout 1800 python -m pytest tests -m gpu -q > gpurun_out/v1_gpu.log 2>&1; echo pytest rc=$?
tail -3 gpurun_out/v1_gpu.log
timeout 400 python bench.py > gpurun_out/v1_bench.log 2>&1; echo bench rc=$?
tail -1 gpurun_out/v1_bench.log
STEPS=5 timeout 900 bash scripts/bench_all.sh > gpurun_out/v1_ball.txt 2>&1
cat gpurun_out/v1_ball.txt

# GPU suite (or a subset: FILES="tests/x.py ..."), log under gpurun_out/
mkdir -p gpurun_out
timeout ${TMO:-1500} python -m pytest ${FILES:-tests} -m gpu -q ${PYTEST_ARGS:-} > gpurun_out/${TAG:-gt}_gpu.log 2>&1; echo pytest rc=$?
tail -5 gpurun_out/${TAG:-gt}_gpu.log

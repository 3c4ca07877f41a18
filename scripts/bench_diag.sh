#!/bin/bash
for i in 1 2; do
python bench.py --steps 8 --warmup 3 --no-cpu-baseline ${BENCH_ARGS} > gpurun_out/diag.json 2>/dev/null
python - <<'PY'
import json
j=json.load(open("gpurun_out/diag.json"))
for k in ("step_ms","step_dp_ms","step_lib_wall_ms","e2e_step_ms"): print(f"{k:18s}", j[k])
print("fill_ms", round(j["roofline"]["fill_ms_per_step"],3), "value %.3e"%j["value"], "e2e %.3e"%j["e2e"]["value"], j["clocks"])
PY
done

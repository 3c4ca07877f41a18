#!/bin/bash
# one bench line per workload (short runs), written to gpurun_out/wl_<name>.json
for wl in "$@"; do
  timeout 900 python bench.py --workload $wl --steps 2 --warmup 1 --no-cpu-baseline > gpurun_out/wl_$wl.json 2> gpurun_out/wl_$wl.err
  python - "$wl" <<'PY'
import json,sys
wl=sys.argv[1]
try:
    t=open(f"gpurun_out/wl_{wl}.json").read(); j=json.loads(t[t.index("{"):])
    r=j["roofline"]
    print(f"{wl:9s} solve={j['ms_per_step']:9.2f} ms  relax/s={j['value']:.3e}  fill={r['fill_ms_per_step']:9.2f} ms fill_relax/s={r['fill_relax_per_s']:.3e} frac={r['frac']:.3f} probes={j['solve']['probes']} dps={j['solve']['unique_dps']} sigma_max={j['solve']['sigma_max']:.3e}")
except Exception as e:
    print(wl, "FAILED", e, open(f"gpurun_out/wl_{wl}.err").read()[-800:])
PY
done

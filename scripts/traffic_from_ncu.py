"""profiles/traffic.json entry from an ncu_summarize metrics file (the DRAM bytes
of the longest level-fill launch; bench.py reports them as roofline.traffic):
python scripts/traffic_from_ncu.py <workload> <metrics.json> <summary.md path as cited>"""
import json, os, sys

wl, mf, cite = sys.argv[1], sys.argv[2], sys.argv[3]
M = json.load(open(mf))
def val(k):
    v, u = M[k][0], M[k][1]
    v = float(str(v).replace(",", ""))
    return v * {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9, "us": 1e-6, "ms": 1e-3, "ns": 1e-9, "s": 1}.get(u, 1)
b = val("dram__bytes_read.sum") + val("dram__bytes_write.sum")
d = val("gpu__time_duration.sum")
peak = json.load(open("MEASURED_PEAKS.json"))["hbm_gbs"]
name = M["Kernel Name"][0][:120]
tf = "profiles/traffic.json"
T = json.load(open(tf)) if os.path.exists(tf) else {}
T[wl] = {"source": f"{cite} (ncu --set full, longest level-fill launch of the workload's largest DP, {name})",
         "dram_bytes_per_launch": b, "duration_s": d, "dram_gbs": b / d / 1e9,
         "dram_frac_of_measured_peak": b / d / 1e9 / peak,
         "l2_hit_pct": float(M["lts__t_sector_hit_rate.pct"][0])}
json.dump(T, open(tf, "w"), indent=1)
print(wl, T[wl])

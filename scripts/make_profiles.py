"""Summarise ncu captures into profiles/ (run here, no GPU)."""
import csv, json, os, subprocess, sys, collections
import numpy as np

def raw(rep):
    out = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
    rows = list(csv.reader(out.splitlines()))
    return dict(zip(rows[0], rows[2])), dict(zip(rows[0], rows[1]))

def val(v, u, k):
    x = float(v[k].replace(",", ""))
    unit = u.get(k, "")
    return x * {"Gbyte": 1e9, "Mbyte": 1e6, "Kbyte": 1e3, "byte": 1, "ms": 1e3, "us": 1, "ns": 1e-3}.get(unit, 1)

KEYS = ["gpu__time_duration.sum", "dram__bytes_read.sum", "dram__bytes_write.sum",
        "dram__throughput.avg.pct_of_peak_sustained_elapsed", "lts__t_sector_hit_rate.pct",
        "l1tex__t_sector_hit_rate.pct", "sm__issue_active.avg.pct_of_peak_sustained_elapsed",
        "sm__warps_active.avg.pct_of_peak_sustained_active", "smsp__inst_executed.sum",
        "launch__registers_per_thread", "launch__grid_size", "l1tex__t_requests_pipe_lsu_mem_global_op_ld.sum",
        "l1tex__t_sectors_pipe_lsu_mem_global_op_ld.sum", "sm__inst_executed_pipe_alu.avg.pct_of_peak_sustained_active",
        "sm__inst_executed_pipe_lsu.avg.pct_of_peak_sustained_active"]

def launches(csvf):
    rows = [r for r in csv.DictReader(l for l in open(csvf) if not l.startswith("=="))]
    tot = collections.defaultdict(float); cnt = collections.Counter()
    for r in rows:
        k = r["Kernel Name"].split("(")[0]
        tot[k] += float(r["Metric Value"].replace(",", "")) / 1e3; cnt[k] += 1
    return tot, cnt

if __name__ == "__main__":
    tag, wl, relax, rows_lvl, W = sys.argv[1], sys.argv[2], float(sys.argv[3]), float(sys.argv[4]), float(sys.argv[5])
    rep = f"gpurun_out/{tag}_full.ncu-rep"
    v, u = raw(rep)
    metrics = {k: [v.get(k), u.get(k)] for k in KEYS}
    json.dump(metrics, open(f"profiles/{tag}_row_fill_{wl}_metrics.json", "w"), indent=1)
    t_us = val(v, u, "gpu__time_duration.sum")
    dram = val(v, u, "dram__bytes_read.sum") + val(v, u, "dram__bytes_write.sum")
    alg = relax + rows_lvl * W
    tot, cnt = launches(f"gpurun_out/{tag}_launches.csv")
    T = sum(tot.values())
    lines = [f"## {tag}: {wl}", "",
             f"Longest level-fill launch (ncu --set full, cold caches, serialised): {t_us:.1f} us, "
             f"{relax:.3g} relaxations ({relax / (t_us * 1e-6):.3g} relax/s), algorithmic bytes {alg:.3g}, "
             f"DRAM read+write {dram:.3g} B (traffic/alg = {dram / alg:.2f}).", "",
             "| metric | value |", "|---|---|"]
    for k in KEYS:
        lines.append(f"| {k} | {v.get(k)} {u.get(k, '')} |")
    lines += ["", "Launch list of one solve (ncu gpu__time_duration, share of device time):", "",
              "| kernel | launches | total us | share |", "|---|---|---|---|"]
    for k in sorted(tot, key=lambda k: -tot[k]):
        lines.append(f"| `{k[-60:]}` | {cnt[k]} | {tot[k]:.1f} | {tot[k] / T:.3f} |")
    open(f"profiles/{tag}_{wl}.md", "w").write("\n".join(lines) + "\n")
    os.system(f"cp gpurun_out/{tag}_launches.csv profiles/{tag}_{wl}_launches.csv")
    tj = json.load(open("profiles/traffic.json")) if os.path.exists("profiles/traffic.json") else {}
    tj[wl] = {"source": f"profiles/{tag}_row_fill_{wl}_metrics.json (ncu --set full, longest row_fill launch of one {wl} solve)",
              "dram_bytes_per_launch": dram, "alg_bytes_per_launch": alg, "traffic_over_alg": dram / alg}
    json.dump(tj, open("profiles/traffic.json", "w"), indent=1)
    print("\n".join(lines[:4]))

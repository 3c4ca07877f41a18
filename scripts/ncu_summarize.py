"""Summarise an ncu capture made by scripts/ncu_top.sh (runs where the report is):
python scripts/ncu_summarize.py <tag> <workload>
-> gpurun_out/<tag>_summary.md (key metrics of the longest level-fill launch, stall
   reasons, hottest SASS, launch list of one solve with shares) and
   gpurun_out/<tag>_metrics.json."""
import collections, csv, json, os, subprocess, sys

tag, wl = sys.argv[1], sys.argv[2]
rep = f"gpurun_out/{tag}_full.ncu-rep"
peak = json.load(open("MEASURED_PEAKS.json"))["hbm_gbs"] if os.path.exists("MEASURED_PEAKS.json") else 6456.2


def ncu(*a):
    return subprocess.run(["ncu", "-i", rep, *a], capture_output=True, text=True).stdout


raw = list(csv.reader(ncu("--page", "raw", "--csv").splitlines()))
h, units, v = raw[0], raw[1], raw[2]
M = {h[i]: (v[i], units[i]) for i in range(len(h))}


def num(k):
    x, u = M.get(k, ("", ""))
    try:
        f = float(str(x).replace(",", ""))
    except ValueError:
        return None
    return f * {"Gbyte": 1e9, "Mbyte": 1e6, "Kbyte": 1e3, "byte": 1, "ms": 1e-3, "us": 1e-6, "ns": 1e-9,
                "msecond": 1e-3, "usecond": 1e-6, "nsecond": 1e-9, "Tbyte/s": 1e12, "Gbyte/s": 1e9,
                "Mbyte/s": 1e6, "byte/s": 1}.get(u, 1)


KEYS = ["Kernel Name", "gpu__time_duration.sum", "dram__bytes_read.sum", "dram__bytes_write.sum",
        "dram__bytes.sum.per_second", "dram__throughput.avg.pct_of_peak_sustained_elapsed",
        "lts__t_sector_hit_rate.pct", "l1tex__t_sector_hit_rate.pct", "sm__issue_active.avg.pct_of_peak_sustained_elapsed",
        "sm__warps_active.avg.pct_of_peak_sustained_active", "smsp__inst_executed.sum", "launch__registers_per_thread",
        "launch__grid_size", "launch__block_size", "sm__inst_executed_pipe_alu.avg.pct_of_peak_sustained_active",
        "sm__inst_executed_pipe_lsu.avg.pct_of_peak_sustained_active",
        "l1tex__t_sectors_pipe_lsu_mem_global_op_ld.sum", "l1tex__t_requests_pipe_lsu_mem_global_op_ld.sum"]
met = {k: list(M.get(k, (None, None))) for k in KEYS}
dur = num("gpu__time_duration.sum")
dram = (num("dram__bytes_read.sum") or 0) + (num("dram__bytes_write.sum") or 0)
dram_gbs = dram / dur / 1e9 if dur else None
met["derived"] = {"dram_bytes": dram, "duration_s": dur, "dram_gbs": dram_gbs, "peak_gbs": peak,
                  "dram_frac": dram_gbs / peak if dram_gbs else None}
stalls = sorted(((k.replace("smsp__pcsamp_warps_issue_stalled_", ""), float(M[k][0] or 0)) for k in M
                 if k.startswith("smsp__pcsamp_warps_issue_stalled_") and not k.endswith("not_issued")),
                key=lambda x: -x[1])
tot_st = sum(x[1] for x in stalls) or 1
json.dump(met, open(f"gpurun_out/{tag}_metrics.json", "w"), indent=1)

src = list(csv.reader(ncu("--page", "source", "--csv").splitlines()))
hot = []
if len(src) > 2:
    hs = src[1]
    i_s, i_e, i_src = hs.index("Warp Stall Sampling (All Samples)"), hs.index("Instructions Executed"), hs.index("Source")
    data = src[2:]
    S = [float(r[i_s] or 0) for r in data]
    T = sum(S) or 1
    hot = [(100 * S[k] / T, data[k][i_e], data[k][i_src].strip()[:80]) for k in sorted(range(len(data)), key=lambda k: -S[k])[:12]]

rows = [r for r in csv.DictReader(l for l in open(f"gpurun_out/{tag}_launches.csv") if not l.startswith("=="))]
tot = collections.defaultdict(float)
cnt = collections.Counter()
for r in rows:
    k = r["Kernel Name"].split("(")[0]
    tot[k] += float(r["Metric Value"].replace(",", "")) / 1e3
    cnt[k] += 1
T = sum(tot.values()) or 1
L = [f"## {tag}: {wl}", "",
     f"Longest level-fill launch (ncu --set full, --clock-control none, cold caches, serialised): "
     f"`{str(M.get('Kernel Name', ('',))[0])[:110]}`", "",
     f"* duration {dur * 1e6:.1f} us; DRAM read+write {dram / 1e6:.1f} MB = **{dram_gbs:.0f} GB/s = "
     f"{100 * dram_gbs / peak:.1f}% of the measured {peak} GB/s** (ncu dram__throughput "
     f"{M.get('dram__throughput.avg.pct_of_peak_sustained_elapsed', ('?',))[0]} % of its own peak)",
     f"* L2 hit rate {M.get('lts__t_sector_hit_rate.pct', ('?',))[0]} %, L1 hit rate {M.get('l1tex__t_sector_hit_rate.pct', ('?',))[0]} %",
     f"* issue active {M.get('sm__issue_active.avg.pct_of_peak_sustained_elapsed', ('?',))[0]} %, warps active "
     f"{M.get('sm__warps_active.avg.pct_of_peak_sustained_active', ('?',))[0]} %, registers "
     f"{M.get('launch__registers_per_thread', ('?',))[0]}, grid {M.get('launch__grid_size', ('?',))[0]} x "
     f"{M.get('launch__block_size', ('?',))[0]}", "",
     "Stall reasons (share of warp samples): " + ", ".join(f"{k} {100 * x / tot_st:.0f}%" for k, x in stalls[:8]), "",
     "Hottest SASS (share of stall samples, executions):", ""]
L += [f"    {s:5.1f}%  {e:>10}  {t}" for s, e, t in hot]
L += ["", "Launch list of one solve (ncu gpu__time_duration, share of device time):", "",
      "| kernel | launches | total us | share |", "|---|---|---|---|"]
for k in sorted(tot, key=lambda k: -tot[k]):
    L.append(f"| `{k[-70:]}` | {cnt[k]} | {tot[k]:.1f} | {tot[k] / T:.3f} |")
open(f"gpurun_out/{tag}_summary.md", "w").write("\n".join(L) + "\n")
print("\n".join(L[:8]))

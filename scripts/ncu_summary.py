"""Summarise an ncu --set full report: key metrics + hottest SASS (run here, no GPU)."""
import csv
import subprocess
import sys

rep = sys.argv[1]
topn = int(sys.argv[2]) if len(sys.argv) > 2 else 40
raw = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
rows = list(csv.reader(raw.splitlines()))
hdr, units, vals = rows[0], rows[1], rows[2]
keys = ["gpu__time_duration.sum", "smsp__inst_executed.sum", "sm__issue_active.avg.pct_of_peak_sustained_elapsed",
        "sm__warps_active.avg.pct_of_peak_sustained_active", "launch__registers_per_thread", "launch__grid_size",
        "l1tex__t_requests_pipe_lsu_mem_global_op_ld.sum", "l1tex__t_sectors_pipe_lsu_mem_global_op_ld.sum",
        "l1tex__t_sector_hit_rate.pct", "lts__t_sector_hit_rate.pct", "dram__bytes_read.sum", "dram__bytes_write.sum",
        "dram__throughput.avg.pct_of_peak_sustained_elapsed", "sm__inst_executed_pipe_lsu.avg.pct_of_peak_sustained_active",
        "sm__inst_executed_pipe_alu.avg.pct_of_peak_sustained_active",
        "l1tex__data_pipe_lsu_wavefronts_mem_shared.sum", "smsp__inst_executed_op_shfl.sum" ]
for h, u, v in zip(hdr, units, vals):
    if h in keys:
        print(f"{h:70s} {v:>16s} {u}")
for h, u, v in zip(hdr, units, vals):
    if h.startswith("smsp__pcsamp_warps_issue_stalled") and not h.endswith("not_issued"):
        try:
            if float(v.replace(",", "")) > 100:
                print(f"  {h[33:]:50s} {v}")
        except ValueError:
            pass
src = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv"], capture_output=True, text=True).stdout
rows = list(csv.reader(src.splitlines()))
hdr = rows[1]
data = rows[2:]
ia = hdr.index("Instructions Executed")
isrc = hdr.index("Source")
iss = hdr.index("Warp Stall Sampling (All Samples)")
tot = sum(float(r[ia] or 0) for r in data)
tots = sum(float(r[iss] or 0) for r in data)
print("total warp inst", tot, "samples", tots)
top = sorted(data, key=lambda r: -float(r[iss] or 0))[:topn]
for r in sorted(top, key=lambda r: int(r[0], 16)):
    print(f"{r[0][-5:]} inst={float(r[ia])/tot*100:5.2f}% stall={float(r[iss])/tots*100:5.2f}% {r[isrc].strip()[:70]}")

"""Hottest SASS instructions (warp stall samples) of an ncu --set full report:
python scripts/ncu_hot.py <rep> [top] — prints share of samples, executed count
and the instruction, plus sample share per 5% slice of the kernel's code."""
import csv, subprocess, sys
rep = sys.argv[1]
top = int(sys.argv[2]) if len(sys.argv) > 2 else 30
out = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv"], capture_output=True, text=True).stdout
rows = list(csv.reader(out.splitlines()))
hdr = rows[1]
data = rows[2:]
i_s = hdr.index("Warp Stall Sampling (All Samples)")
i_e = hdr.index("Instructions Executed")
i_src = hdr.index("Source")
S = [float(r[i_s] or 0) for r in data]
tot = sum(S) or 1
print(f"{len(data)} SASS lines, {tot:.0f} samples")
for k in sorted(range(len(data)), key=lambda k: -S[k])[:top]:
    print(f"{k:5d} {100 * S[k] / tot:5.1f}%  ex={float(data[k][i_e] or 0):9.0f}  {data[k][i_src].strip()[:90]}")
n = len(data)
sl = max(1, n // 20)
print("slices:", " ".join(f"{a}:{100 * sum(S[a:a + sl]) / tot:.0f}%" for a in range(0, n, sl)))

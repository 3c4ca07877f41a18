"""Instruction share by basic-block-like runs (consecutive SASS lines with the same
execution count) of an ncu --set full report's source page."""
import csv, subprocess, sys
rep = sys.argv[1]
src = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv"], capture_output=True, text=True).stdout
rows = list(csv.reader(src.splitlines()))
hdr = rows[1]; data = rows[2:]
ia = hdr.index("Instructions Executed"); isrc = hdr.index("Source")
tot = sum(float(r[ia] or 0) for r in data)
runs = []
cur = None
for r in data:
    c = float(r[ia] or 0)
    if cur and abs(cur[1] - c) < 1e-9:
        cur[2] += c; cur[3].append(r[isrc].strip()); continue
    cur = [r[0][-5:], c, c, [r[isrc].strip()]]
    runs.append(cur)
runs.sort(key=lambda x: -x[2])
for a, c, t, ins in runs[:int(sys.argv[2]) if len(sys.argv) > 2 else 15]:
    ops = " ".join(i.split()[0] if not i.startswith("@") else i.split()[1] for i in ins[:12])
    print(f"{a} n={len(ins):3d} exec/inst={c:.3g} share={t / tot * 100:5.1f}%  {ops}")

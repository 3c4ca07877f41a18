"""Opcode mix of an ncu --set full report (executed instructions by opcode)."""
import csv, subprocess, sys
from collections import Counter
rep = sys.argv[1]
src = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv"], capture_output=True, text=True).stdout
rows = list(csv.reader(src.splitlines()))
hdr = rows[1]; data = rows[2:]
ia = hdr.index("Instructions Executed"); isrc = hdr.index("Source")
tot = sum(float(r[ia] or 0) for r in data)
c = Counter()
for r in data:
    op = r[isrc].strip().split()
    if not op:
        continue
    o = op[1] if op[0].startswith('@') else op[0]
    c[o.split('.')[0]] += float(r[ia] or 0)
print("total warp inst %.4g" % tot)
for o, v in c.most_common(int(sys.argv[2]) if len(sys.argv) > 2 else 20):
    print(f"{o:12s} {v / tot * 100:5.1f}%")

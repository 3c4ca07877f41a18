"""Host timeline of one solve from PTAS_TRACE=1 stderr (the last solve in the log):
python scripts/timeline.py gpurun_out/x.log"""
import re, sys
lines = open(sys.argv[1]).read().splitlines()
idx = [i for i, l in enumerate(lines) if l.startswith("[ptas] solve |")]
end = idx[-1]
start = idx[-2] + 1 if len(idx) > 1 else 0
seg = lines[start:end + 1]
t0 = float(re.search(r"host clock ([\d.]+)", seg[-1]).group(1))
for l in seg:
    m = re.search(r"host clock ([\d.]+) \.\. ([\d.]+)", l)
    if not m:
        continue
    a, b = float(m.group(1)) - t0, float(m.group(2)) - t0
    print("%8.3f %8.3f  %s" % (a, b, l.split("|")[0][:110]))

"""Launch list (ncu --metrics gpu__time_duration.sum --csv) grouped by kernel:
python scripts/ncu_launches.py <csv> [title] -> markdown table on stdout."""
import collections, csv, sys

rows = [r for r in csv.DictReader(l for l in open(sys.argv[1]) if not l.startswith("=="))]
tot = collections.OrderedDict()
cnt = collections.Counter()
for r in rows:
    if r.get("Metric Name") != "gpu__time_duration.sum":
        continue
    name = r["Kernel Name"].split("(")[0]
    v = float(r["Metric Value"].replace(",", ""))
    scale = {"nsecond": 1e-3, "ns": 1e-3, "usecond": 1.0, "us": 1.0, "msecond": 1e3, "ms": 1e3}[r.get("Metric Unit", "us")]
    tot[name] = tot.get(name, 0.0) + v * scale
    cnt[name] += 1
T = sum(tot.values()) or 1.0
print("## " + (sys.argv[2] if len(sys.argv) > 2 else sys.argv[1]))
print()
print("ncu --metrics gpu__time_duration.sum --clock-control none (serialised, cold caches; the share is what is comparable).")
print()
print("| kernel | launches | total us | share |")
print("|---|---|---|---|")
for k, v in sorted(tot.items(), key=lambda kv: -kv[1]):
    print(f"| `{k}` | {cnt[k]} | {v:.1f} | {v / T:.3f} |")

"""Summarise an ncu --metrics gpu__time_duration.sum launch list (CSV) by kernel."""
import collections
import csv
import sys

rows = list(csv.DictReader(l for l in open(sys.argv[1]) if not l.startswith("==")))
d = collections.defaultdict(list)
for r in rows:
    if r.get("Metric Name") == "gpu__time_duration.sum":
        v = float(r["Metric Value"]) * (1e3 if r.get("Metric Unit") == "usecond" else 1.0)
        d[r["Kernel Name"].split("(")[0][:80]].append(v)
tot = sum(sum(v) for v in d.values())
print(f"{'total_us':>10} {'n':>4} {'avg_us':>9} {'share':>6}  kernel")
for k, v in sorted(d.items(), key=lambda kv: -sum(kv[1])):
    print(f"{sum(v)/1e3:10.1f} {len(v):4d} {sum(v)/len(v)/1e3:9.2f} {sum(v)/tot:6.3f}  {k}")

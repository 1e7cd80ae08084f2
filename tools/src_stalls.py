"""Dev tool: summarise an `ncu --page source --csv --print-source sass` dump
(tools/ncu_source.sh): stall-reason totals and the hottest SASS lines."""
import csv
import sys

rows = list(csv.reader(open(sys.argv[1])))
h = rows[1]
data = [r for r in rows[2:] if len(r) == len(h)]
cols = [c for c in h if c.startswith("stall_") and "Not Issued" not in c]
tot = {c: sum(int(r[h.index(c)]) for r in data if r[h.index(c)].isdigit()) for c in cols}
s = sum(tot.values()) or 1
print(rows[0][1][:100])
print("  ".join(f"{c[6:]} {v / s * 100:.1f}%" for c, v in sorted(tot.items(), key=lambda x: -x[1])[:8]))
ia, isrc, iex = h.index("Warp Stall Sampling (All Samples)"), h.index("Source"), h.index("Instructions Executed")
n = int(sys.argv[2]) if len(sys.argv) > 2 else 25
for r in sorted(data, key=lambda r: -int(r[ia]) if r[ia].isdigit() else 0)[:n]:
    top = max(cols, key=lambda c: int(r[h.index(c)]) if r[h.index(c)].isdigit() else 0)
    print(f"{int(r[ia]) / s * 100:5.1f}% ex={r[iex]:>8s} {top[6:]:>16s}  {r[isrc].strip()[:80]}")

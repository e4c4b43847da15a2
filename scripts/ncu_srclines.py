"""Top SASS lines by warp-stall samples from `ncu --page source --csv` output (first kernel
instance): python scripts/ncu_srclines.py file.csv [top]."""
import csv, sys
rows = list(csv.reader(open(sys.argv[1])))
top = int(sys.argv[2]) if len(sys.argv) > 2 else 30
h = rows[1]
si, src, ie = h.index("Warp Stall Sampling (All Samples)"), h.index("Source"), h.index("Instructions Executed")
data = []
for r in rows[2:]:
    if len(r) <= ie:
        continue
    if r[0] == "Kernel Name":
        break
    data.append((int(r[si]) if r[si].isdigit() else 0, len(data), r[src].strip(), r[ie]))
tot = sum(d[0] for d in data)
print(f"{len(data)} instructions, {tot} samples")
for s, i, t, e in sorted(data, reverse=True)[:top]:
    print(f"{s:6d} {100.0 * s / max(tot, 1):5.1f}% #{i:5d} x{e:>7s}  {t[:80]}")

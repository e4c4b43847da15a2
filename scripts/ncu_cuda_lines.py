"""Aggregate an `ncu --page source --csv --print-source cuda,sass` export by CUDA source line:
warp-stall samples (all), instructions executed and the top stall reasons per line."""
import csv
import sys
from collections import defaultdict

rows = list(csv.reader(open(sys.argv[1], errors="replace")))
top = int(sys.argv[2]) if len(sys.argv) > 2 else 30
agg = defaultdict(lambda: [0.0, 0.0, defaultdict(float), ""])
hdr, fname = None, "?"
f = lambda x: float(x) if x not in ("", "-", None) else 0.0
for r in rows:
    if len(r) >= 2 and r[0] == "File Path":
        fname = r[1].split("/")[-1]
        continue
    if len(r) > 4 and r[0] == "Line No":
        hdr = r
        iW = hdr.index("Warp Stall Sampling (All Samples)")
        iE = hdr.index("Instructions Executed")
        stalls = [(i, h) for i, h in enumerate(hdr) if h.startswith("stall_") and "Not Issued" not in h]
        continue
    if hdr is None or len(r) != len(hdr) or not r[0].isdigit():
        continue
    a = agg[(fname, int(r[0]))]
    a[0] += f(r[iW]); a[1] += f(r[iE]); a[3] = r[1]
    for i, h in stalls:
        a[2][h] += f(r[i])
tot = sum(v[0] for v in agg.values())
print(f"total samples {tot:.0f}")
for (fn, ln), (w, e, st, src) in sorted(agg.items(), key=lambda kv: -kv[1][0])[:top]:
    s3 = ", ".join(f"{k[6:]} {v:.0f}" for k, v in sorted(st.items(), key=lambda kv: -kv[1])[:3] if v > 0)
    print(f"{w:7.0f} {100 * w / max(tot, 1):5.1f}% {e:9.0f}  {fn}:{ln}  {src.strip()[:70]}  [{s3}]")

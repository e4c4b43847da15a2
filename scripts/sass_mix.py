"""Instruction mix (warp-level executed counts and stall samples by opcode) of the first kernel in
an ncu report: python scripts/sass_mix.py report.ncu-rep"""
import collections, csv, subprocess, sys
out = subprocess.run(["ncu", "-i", sys.argv[1], "--page", "source", "--csv"], capture_output=True, text=True).stdout
rows = list(csv.reader(out.splitlines()))
hdr = rows[1]
data = [r for r in rows[2:] if len(r) >= len(hdr) - 1]
iS, iW, iE = hdr.index("Source"), hdr.index("Warp Stall Sampling (All Samples)"), hdr.index("Instructions Executed")
f = lambda x: float(x) if x not in ("", "-") else 0.0
tot = sum(f(r[iE]) for r in data); totw = sum(f(r[iW]) for r in data) or 1
print(rows[0][1][:90], f"warp-instructions {tot:.0f}")
op, st = collections.Counter(), collections.Counter()
for r in data:
    t = r[iS].split()
    if not t:
        continue
    o = (t[1] if t[0].startswith("@") else t[0]).split(".")[0]
    op[o] += f(r[iE]); st[o] += f(r[iW])
for o, c in op.most_common(int(sys.argv[2]) if len(sys.argv) > 2 else 14):
    print(f"{o:10s} {c:12.0f} {c / tot * 100:5.1f}%  stall {st[o] / totw * 100:5.1f}%")

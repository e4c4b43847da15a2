"""Top stall lines of an `ncu --page source --csv` export (first kernel section)."""
import csv, sys
rows = list(csv.reader(open(sys.argv[1])))
n = int(sys.argv[2]) if len(sys.argv) > 2 else 25
starts = [i for i, r in enumerate(rows) if len(r) > 2 and r[1] == 'Source'] + [len(rows)]
for a, b in zip(starts[:-1], starts[1:]):
    hdr = rows[a]
    data = [r for r in rows[a + 1:b] if len(r) == len(hdr)]
    iS, iW, iE = hdr.index('Source'), hdr.index('Warp Stall Sampling (All Samples)'), hdr.index('Instructions Executed')
    f = lambda x: float(x) if x not in ('', '-') else 0.0
    tot = sum(f(r[iW]) for r in data)
    print(f"--- section rows={len(data)} samples={tot:.0f} instructions={sum(f(r[iE]) for r in data):.0f}")
    for r in sorted(data, key=lambda r: -f(r[iW]))[:n]:
        print(f"{f(r[iW]):7.0f} {f(r[iE]):8.0f}  {r[iS].strip()[:110]}")
    break

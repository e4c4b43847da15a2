"""Stall samples per CUDA source line from two `ncu --page source --csv` exports of one kernel:
--print-source sass (per-instruction metrics) and --print-source cuda,sass (line <-> address map)."""
import collections, csv, sys

sass, mix = sys.argv[1], sys.argv[2]
n = int(sys.argv[3]) if len(sys.argv) > 3 else 25
rows = list(csv.reader(open(sass)))
hdr = rows[1]
iA, iW = hdr.index('Address'), hdr.index('Warp Stall Sampling (All Samples)')
data = [r for r in rows[2:] if len(r) == len(hdr)]
addr2line, cur, fpath = {}, None, None
for r in csv.reader(open(mix)):
    if r and r[0] == 'File Path':
        fpath = r[1].split('/')[-1]
    if len(r) >= 4:
        if r[0] and r[0] != 'Line No':
            cur = (fpath, r[0], r[1][:90])
        if r[2].startswith('0x'):
            addr2line[r[2]] = cur
agg = collections.Counter()
for r in data:
    agg[addr2line.get(r[iA])] += float(r[iW] or 0)
tot = sum(agg.values())
print(f"total samples {tot:.0f}")
for k, v in agg.most_common(n):
    print(f"{v:7.0f} {100 * v / max(tot, 1):5.1f}% {k}")

"""Summarise an ncu --csv launch list (skips the ==PROF== preamble): mean per kernel."""
import collections, csv, io, sys
txt = open(sys.argv[1]).read().splitlines()
start = next(i for i, l in enumerate(txt) if l.startswith('"ID"'))
rows = list(csv.DictReader(io.StringIO("\n".join(txt[start:]))))
agg = collections.OrderedDict()
for r in rows:
    k = r["Kernel Name"].split("(")[0][:48]
    m = r["Metric Name"]; v = float(r["Metric Value"].replace(",", ""))
    agg.setdefault(k, collections.defaultdict(list))[m].append(v)
tot = 0.0
for k, d in agg.items():
    t = d.get("gpu__time_duration.sum", [0]); rd = d.get("dram__bytes_read.sum", [0]); wr = d.get("dram__bytes_write.sum", [0])
    tt = sum(t) / len(t) / 1e3; tot += tt
    print(f"{k:48s} n={len(t):3d} t_us={tt:9.2f} read_MB={sum(rd)/len(rd)/1e6:9.2f} write_MB={sum(wr)/len(wr)/1e6:8.2f} GB/s={(sum(rd)+sum(wr))/len(rd)/(tt*1e3) if tt else 0:8.1f}")
print(f"sum of per-kernel means: {tot:.1f} us")

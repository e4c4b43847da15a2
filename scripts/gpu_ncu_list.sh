mkdir -p gpurun_out
timeout 600 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none -s 200 -c 60 --csv --log-file gpurun_out/launches.csv python bench.py --steps 20 --warmup 20 --no-e2e --no-cpu-baseline > gpurun_out/ncu_bench.log 2>&1
tail -3 gpurun_out/ncu_bench.log
python - <<'PY'
import csv, collections
rows = list(csv.DictReader(open("gpurun_out/launches.csv")))
agg = collections.OrderedDict()
for r in rows:
    k = r["Kernel Name"].split("(")[0][:60]
    m = r["Metric Name"]; v = float(r["Metric Value"].replace(",", ""))
    agg.setdefault(k, collections.defaultdict(list))[m].append(v)
for k, d in agg.items():
    t = d.get("gpu__time_duration.sum", [0]); rd = d.get("dram__bytes_read.sum", [0]); wr = d.get("dram__bytes_write.sum", [0])
    print(f"{k:60s} n={len(t):3d} t_us={sum(t)/len(t)/1e3:9.2f} read_MB={sum(rd)/len(rd)/1e6:9.2f} write_MB={sum(wr)/len(wr)/1e6:8.2f}")
PY

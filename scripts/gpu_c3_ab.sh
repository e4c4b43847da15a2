# C3 (nb = 20): scalar k_response vs the DMMA k_response_mma for one slice, plus a launch list
mkdir -p gpurun_out
for c in C3 C2 C4; do
  for mma in 0 1; do
    if [ $mma = 1 ]; then export EFIT_RESP_MMA=1; else unset EFIT_RESP_MMA; fi
    timeout 300 python bench.py --config $c --steps 500 --warmup 10 --no-cpu-baseline 2>&1 | tail -1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('$c mma=$mma', d['value'], d['config']['step_breakdown_us'])" || echo "$c $mma failed"
  done
done
unset EFIT_RESP_MMA
timeout 300 ncu --metrics gpu__time_duration.sum --clock-control none -s 200 -c 60 --csv --log-file gpurun_out/c3_launches.csv python bench.py --config C3 --steps 5 --warmup 5 --no-e2e --no-cpu-baseline > /dev/null 2>&1
python - <<'PY'
import csv, collections
t = collections.defaultdict(list)
for r in csv.DictReader(l for l in open('gpurun_out/c3_launches.csv') if not l.startswith('==')):
    if r.get('Metric Name') == 'gpu__time_duration.sum':
        t[r['Kernel Name'][:60]].append(float(r['Metric Value']))
for k, v in sorted(t.items(), key=lambda kv: -sum(kv[1])):
    print(f"{k:60s} n={len(v):3d} avg={sum(v)/len(v)/1000:8.2f} us")
PY

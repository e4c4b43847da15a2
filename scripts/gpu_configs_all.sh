# every BASELINE config through bench.py (one GPU): it/s and the per-step breakdown
mkdir -p gpurun_out
for c in C1 C2 C3 C4 C5; do
  for m in sym table; do
    timeout 300 python bench.py --config $c --steps 500 --warmup 10 --no-cpu-baseline --mode $m 2>&1 | tail -1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('$c $m', d['value'], d['e2e']['value'], d['config']['step_breakdown_us'], d['roofline']['frac'])" || echo "$c $m failed"
  done
done

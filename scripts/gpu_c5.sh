# 1025^2 stress case: sampled parity, then bench in sym / table / otf-sym
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_parity.py -x -q -k c5 2>&1 | tail -3
for m in sym table otf-sym; do
  timeout 300 python bench.py --config C5 --steps 100 --warmup 5 --no-cpu-baseline --no-e2e --mode $m 2>&1 | tail -1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('C5 $m', d['value'], d['config'].get('step_breakdown_us'), d['roofline']['achieved'], d['roofline']['frac'], d['config']['init_s'])" || echo "C5 $m failed"
done

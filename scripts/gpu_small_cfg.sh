# small-grid response row split: tests + C1/C2/C3/C4 sym bench
mkdir -p gpurun_out
timeout 900 python -m pytest tests -m gpu -x -q 2>&1 | tail -2
for c in C1 C2 C3 C4; do
timeout 300 python bench.py --config $c --steps 1000 --warmup 10 --no-cpu-baseline --no-e2e 2>&1 | tail -1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('$c', d['value'], d['config']['step_breakdown_us'])" || echo "$c failed"
done

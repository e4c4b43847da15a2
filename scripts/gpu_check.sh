# Re-entry check: tests, smoke, default bench, per-mode bench
mkdir -p gpurun_out
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,memory.total --format=csv
timeout 900 python -m pytest tests -m gpu -x -q 2>&1 | tail -30
timeout 300 python __graft_entry__.py --smoke 2>&1 | tail -3
timeout 600 python bench.py 2>&1 | tail -1 | tee gpurun_out/bench_default.json
for m in table sym otf; do
  timeout 300 python bench.py --steps 500 --warmup 20 --no-cpu-baseline --no-e2e --mode $m > gpurun_out/bench_$m.log 2>&1
  tail -1 gpurun_out/bench_$m.log | python -c "import json,sys; d=json.loads(sys.stdin.read()); print(d['config'].get('green_mode'), d['value'], d['config'].get('step_breakdown_us'), d['roofline']['achieved'], d['roofline']['frac'])"
done

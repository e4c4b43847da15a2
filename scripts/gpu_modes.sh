timeout 900 python -m pytest tests -m gpu -x -q 2>&1 | tail -3
for i in 1 2; do
timeout 300 python bench.py --steps 3000 --warmup 50 --no-e2e --no-cpu-baseline --no-profile 2>&1 | python -c "import json,sys; d=json.loads(sys.stdin.readlines()[-1]); print('graph', d['value'], d['ms_per_step'])"
timeout 300 python bench.py --steps 3000 --warmup 50 --no-e2e --no-cpu-baseline 2>&1 | python -c "import json,sys; d=json.loads(sys.stdin.readlines()[-1]); print('profiled', d['value'], d['ms_per_step'], d['config']['step_breakdown_us'], d['roofline']['frac'])"
done

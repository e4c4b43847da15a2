# f3: edge-case tests + staged-limiter final kernel timing
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_steps.py -x -q 2>&1 | tail -4
timeout 600 python bench.py --rule full --steps 300 --no-cpu-baseline --no-e2e > gpurun_out/f3f_bench.json 2>&1; tail -1 gpurun_out/f3f_bench.json | python -c "import json,sys; d=json.loads(sys.stdin.read()); print(d['value'], d['config']['step_breakdown_us'])"
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -s 300 -c 54 --csv --log-file gpurun_out/f3f_launches.csv python bench.py --rule full --steps 20 --warmup 30 --reps 1 --no-e2e --no-cpu-baseline --no-profile > /dev/null 2>&1
python scripts/ncu_summarize.py gpurun_out/f3f_launches.csv 2>&1 | grep -i 'steps'

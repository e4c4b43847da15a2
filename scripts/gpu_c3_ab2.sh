# new response-kernel choice: parity of both kernels, all configs, C3 launch list
mkdir -p gpurun_out
timeout 900 python -m pytest tests -m gpu -q 2>&1 | tail -3
timeout 300 python __graft_entry__.py --smoke 2>&1 | tail -1
for c in C1 C2 C3 C4; do
  timeout 300 python bench.py --config $c --steps 500 --warmup 10 --no-cpu-baseline 2>&1 | tail -1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('$c', d['value'], d['e2e']['value'], d['config']['step_breakdown_us'])" || echo "$c failed"
done
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -s 200 -c 60 --csv --log-file gpurun_out/c3_launches.csv python bench.py --config C3 --steps 20 --warmup 20 --no-e2e --no-cpu-baseline > gpurun_out/ncu_c3.log 2>&1
python scripts/ncu_summarize.py gpurun_out/c3_launches.csv

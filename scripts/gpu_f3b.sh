# f3 after the restructure: tests, bench, launch list
mkdir -p gpurun_out
timeout 600 python -m pytest tests/test_gpu_steps.py -x -q 2>&1 | tail -15
for c in C4 C5; do timeout 600 python bench.py --rule full --config $c --steps 300 --no-cpu-baseline --no-e2e > gpurun_out/f3c_bench_$c.json 2>&1; tail -1 gpurun_out/f3c_bench_$c.json | python -c "import json,sys; d=json.loads(sys.stdin.read()); print(d['value'], d['config']['step_breakdown_us'])"; done
timeout 900 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none -s 300 -c 54 --csv --log-file gpurun_out/f3c_launches_c4.csv python bench.py --rule full --steps 20 --warmup 30 --reps 1 --no-e2e --no-cpu-baseline --no-profile > gpurun_out/f3c_ncu_list.log 2>&1
python scripts/ncu_summarize.py gpurun_out/f3c_launches_c4.csv 2>&1 | grep -i 'steps\|sum'

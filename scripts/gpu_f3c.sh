# f3 fill v3: tests, bench, launch list, ncu source of final/fill
mkdir -p gpurun_out
timeout 600 python -m pytest tests/test_gpu_steps.py -x -q 2>&1 | tail -5
for c in C4 C5; do timeout 600 python bench.py --rule full --config $c --steps 300 --no-cpu-baseline --no-e2e > gpurun_out/f3d_bench_$c.json 2>&1; tail -1 gpurun_out/f3d_bench_$c.json | python -c "import json,sys; d=json.loads(sys.stdin.read()); print(d['value'], d['config']['step_breakdown_us'])"; done
timeout 900 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none -s 300 -c 54 --csv --log-file gpurun_out/f3d_launches_c4.csv python bench.py --rule full --steps 20 --warmup 30 --reps 1 --no-e2e --no-cpu-baseline --no-profile > gpurun_out/f3d_ncu_list.log 2>&1
python scripts/ncu_summarize.py gpurun_out/f3d_launches_c4.csv 2>&1 | grep -i 'steps\|sum'
timeout 900 ncu --set full --clock-control none --import-source on -k "regex:k_steps_f" -s 20 -c 2 -o gpurun_out/f3d_full -f python bench.py --rule full --steps 4 --warmup 10 --reps 1 --no-e2e --no-cpu-baseline --no-profile > gpurun_out/f3d_ncu_full.log 2>&1
for k in k_steps_final k_steps_fill; do
  python scripts/ncu_details.py gpurun_out/f3d_full.ncu-rep $k > gpurun_out/f3d_full_$k.txt 2>&1
  ncu -i gpurun_out/f3d_full.ncu-rep --page source --csv --print-source cuda -k regex:$k > gpurun_out/f3d_src_$k.csv 2>/dev/null
done
rm -f gpurun_out/*.ncu-rep

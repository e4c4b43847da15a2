# ncu --set full (+ source) of the f3 steps_ kernels at C4 (diverted twin), after a clean bench run
mkdir -p gpurun_out
timeout 600 python -m pytest tests/test_gpu_steps.py -x -q 2>&1 | tail -3
timeout 600 python bench.py --rule full --steps 200 --no-cpu-baseline --no-e2e > gpurun_out/f3b_bench.json 2>&1; tail -1 gpurun_out/f3b_bench.json | python -c "import json,sys; d=json.loads(sys.stdin.read()); print(d['value'], d['config']['step_breakdown_us'])"
timeout 900 ncu --set full --clock-control none --import-source on -k "regex:k_steps_" -s 30 -c 3 -o gpurun_out/f3_full -f python bench.py --rule full --steps 4 --warmup 10 --reps 1 --no-e2e --no-cpu-baseline --no-profile > gpurun_out/f3_ncu_full.log 2>&1
tail -2 gpurun_out/f3_ncu_full.log
for k in k_steps_scan k_steps_fill k_steps_bits; do
  python scripts/ncu_details.py gpurun_out/f3_full.ncu-rep $k > gpurun_out/f3_full_$k.txt 2>&1
  ncu -i gpurun_out/f3_full.ncu-rep --page source --csv -k regex:$k > gpurun_out/f3_src_$k.csv 2>/dev/null
  python scripts/ncu_srclines.py gpurun_out/f3_src_$k.csv 30 > gpurun_out/f3_srctop_$k.txt 2>&1
done
rm -f gpurun_out/*.ncu-rep gpurun_out/f3_src_*.csv

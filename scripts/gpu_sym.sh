# SYM-mode bring-up: GPU parity tests, then bench in table and sym modes, then one ncu capture
mkdir -p gpurun_out
timeout 900 python -m pytest tests -m gpu -x -q 2>&1 | tail -30
for m in table sym; do
  timeout 300 python bench.py --steps 1000 --warmup 20 --no-cpu-baseline --no-e2e --mode $m > gpurun_out/bench_$m.log 2>&1
  tail -1 gpurun_out/bench_$m.log | python -c "import json,sys; d=json.loads(sys.stdin.read()); print(d['config']['green_mode'], d['value'], d['config']['step_breakdown_us'], d['roofline']['achieved'], d['roofline']['frac'])"
done
timeout 600 ncu --set full --clock-control none --import-source on -k "regex:k_bnd_sym|k_response" -s 20 -c 2 -o gpurun_out/sym_full python bench.py --steps 4 --warmup 30 --no-e2e --no-cpu-baseline --mode sym > gpurun_out/ncu_sym.log 2>&1
tail -3 gpurun_out/ncu_sym.log

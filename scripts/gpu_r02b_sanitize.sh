# compute-sanitizer over every per-iteration kernel incl. the f3 steps_ kernels (33^2), + f3 tests
mkdir -p gpurun_out
timeout 600 python -m pytest tests/test_gpu_steps.py tests/test_gpu_multi.py -x -q 2>&1 | tail -3
for tool in memcheck racecheck synccheck initcheck; do
  timeout 900 compute-sanitizer --tool $tool --print-limit 20 python scripts/sanitize_small.py 33 > gpurun_out/r02b_sanitize_$tool.txt 2>&1
  echo "$tool rc=$?: $(tail -2 gpurun_out/r02b_sanitize_$tool.txt | tr '\n' ' ')"
done
timeout 600 python bench.py --rule full --steps 300 --no-cpu-baseline --no-e2e > gpurun_out/f3e_bench.json 2>&1; tail -1 gpurun_out/f3e_bench.json | python -c "import json,sys; d=json.loads(sys.stdin.read()); print(d['value'], d['config']['step_breakdown_us'])"

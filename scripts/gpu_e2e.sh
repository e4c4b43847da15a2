# e2e whole-call graph: fit_host tests + default bench (e2e)
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_multi.py -x -q -k fit_host 2>&1 | tail -3
timeout 600 python bench.py --no-cpu-baseline > gpurun_out/e2e_bench.json 2>gpurun_out/e2e_bench.err; tail -1 gpurun_out/e2e_bench.json | python -c "import json,sys; d=json.loads(sys.stdin.read()); print(d['value'], d['e2e'], d['config']['step_breakdown_us'])"; tail -3 gpurun_out/e2e_bench.err

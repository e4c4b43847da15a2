# the scaling run's sharded step (NCCL exchange, graph-captured) exercised on one GPU (world of 1)
mkdir -p gpurun_out
for m in sym table; do
timeout 300 python bench.py --sharded --steps 500 --warmup 10 --no-cpu-baseline --mode $m 2>&1 | tail -1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('sharded $m', d['value'], d['e2e'], d['gpu_launches'])"
done
timeout 300 python bench.py --steps 500 --warmup 10 --no-cpu-baseline 2>&1 | tail -1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('single', d['value'], d['e2e'], d['gpu_launches'])"

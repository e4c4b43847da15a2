# the scaling run's sharded step (NCCL exchange, graph-captured) exercised on one GPU (world of 1)
mkdir -p gpurun_out
for m in sym table; do
timeout 300 python bench.py --sharded --steps 500 --warmup 10 --no-cpu-baseline --mode $m 2>&1 | tail -1 | cut -c1-1200
done
timeout 300 python -m torch.distributed.run --nnodes=1 --nproc-per-node 1 --master-addr 127.0.0.1 --master-port 29541 bench.py --gpus 1 --steps 200 --warmup 5 --no-cpu-baseline 2>&1 | tail -1 | cut -c1-300

mkdir -p gpurun_out
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv
timeout 600 python bench.py --steps 2000 --warmup 20 2>&1 | tail -5
timeout 300 python bench.py --steps 200 --warmup 5 --no-cpu-baseline --no-e2e --mode otf 2>&1 | tail -3

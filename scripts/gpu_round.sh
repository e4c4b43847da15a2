# tests + smoke + bench in one box session
mkdir -p gpurun_out
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,memory.total --format=csv
timeout 900 python -m pytest tests -m gpu -x -q 2>&1 | tail -30
timeout 300 python __graft_entry__.py --smoke 2>&1 | tail -3
timeout 600 python bench.py 2>&1 | tail -2 | tee gpurun_out/bench_default.json

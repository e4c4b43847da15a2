mkdir -p gpurun_out
set -x
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,memory.total --format=csv
nproc
timeout 900 python -m pytest tests -m gpu -x -q 2>&1 | tail -60
timeout 300 python __graft_entry__.py --smoke 2>&1 | tail -5

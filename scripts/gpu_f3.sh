# f3 (full steps_) GPU parity + quick timing of the normalisation
mkdir -p gpurun_out
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv
timeout 1200 python -m pytest tests/test_gpu_steps.py -x -q 2>&1 | tail -30 | tee gpurun_out/f3_tests.txt
timeout 900 python -m pytest tests -m gpu -x -q 2>&1 | tail -5 | tee gpurun_out/f3_alltests.txt

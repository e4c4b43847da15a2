# f4 fused variant: batch tests (incl. boundary_basis), full GPU suite, trade-off measurement
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_batch.py -x -q 2>&1 | tail -3
timeout 900 python -m pytest tests -m gpu -x -q 2>&1 | tail -2
timeout 300 python scripts/measure_f4.py 2>&1 | tail -1
CFG=C2 timeout 300 python scripts/measure_f4.py 2>&1 | tail -1

# round-end self-check: GPU tests, smoke, default bench, batch bench, reference arm
mkdir -p gpurun_out
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv,noheader
timeout 900 python -m pytest tests -m gpu -q 2>&1 | tail -2
timeout 300 python __graft_entry__.py --smoke 2>&1 | tail -1
timeout 600 python bench.py 2>&1 | tail -1 > gpurun_out/r01_bench_final.json; cut -c1-400 gpurun_out/r01_bench_final.json
timeout 600 python bench.py --slices 8 --steps 400 2>&1 | tail -1 > gpurun_out/r01_bench_s8.json; cut -c1-300 gpurun_out/r01_bench_s8.json
timeout 600 python bench.py --impl reference --steps 20 --warmup 1 2>&1 | tail -1 > gpurun_out/r01_bench_reference.json; cut -c1-300 gpurun_out/r01_bench_reference.json

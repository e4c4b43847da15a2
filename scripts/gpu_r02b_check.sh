# Round-2 re-entry check after the k_bnd_sym ring change: GPU tests, smoke, default bench
mkdir -p gpurun_out
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,memory.total --format=csv
timeout 1500 python -m pytest tests -m gpu -x -q 2>&1 | tail -30 | tee gpurun_out/r02b_gputests.txt
timeout 300 python __graft_entry__.py --smoke 2>&1 | tail -3
timeout 600 python bench.py > gpurun_out/r02b_bench_default.json 2> gpurun_out/r02b_bench_default.err
tail -1 gpurun_out/r02b_bench_default.json

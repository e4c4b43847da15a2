# tests + bench + ncu launch list in one box session
mkdir -p gpurun_out
timeout 900 python -m pytest tests -m gpu -x -q 2>&1 | tail -15
timeout 600 python bench.py --steps 2000 --warmup 20 ${BENCH_ARGS} 2>&1 | tail -2
timeout 600 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none -s 200 -c 60 --csv --log-file gpurun_out/launches.csv python bench.py --steps 20 --warmup 20 --no-e2e --no-cpu-baseline > gpurun_out/ncu_bench.log 2>&1
python scripts/ncu_summarize.py gpurun_out/launches.csv

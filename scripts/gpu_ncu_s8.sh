mkdir -p gpurun_out
timeout 600 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none -s 400 -c 200 --csv --log-file gpurun_out/r01_launches_s8.csv python bench.py --steps 10 --warmup 10 --slices 8 --no-cpu-baseline > gpurun_out/ncu_s8.log 2>&1
python scripts/ncu_summarize.py gpurun_out/r01_launches_s8.csv

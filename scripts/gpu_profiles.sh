# round profiles: launch list (cold, serialised), warm-cache launch list, full sets of the two HBM kernels
mkdir -p gpurun_out
timeout 600 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none -s 300 -c 45 --csv --log-file gpurun_out/r01_launches_cold.csv python bench.py --steps 20 --warmup 30 --no-e2e --no-cpu-baseline > /dev/null 2>&1
timeout 600 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --cache-control none --clock-control none -s 300 -c 45 --csv --log-file gpurun_out/r01_launches_warm.csv python bench.py --steps 20 --warmup 30 --no-e2e --no-cpu-baseline > /dev/null 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k "regex:k_bnd_tb|k_response" -s 20 -c 2 -o gpurun_out/r01_full -f python bench.py --steps 4 --warmup 30 --no-e2e --no-cpu-baseline > gpurun_out/r01_full.log 2>&1
tail -2 gpurun_out/r01_full.log
ls -la gpurun_out | head

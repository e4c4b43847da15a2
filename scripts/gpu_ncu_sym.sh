# ncu --set full of the two HBM streams in sym mode (k_bnd_sym, k_response) + the table-mode k_bnd_tb
mkdir -p gpurun_out
timeout 900 ncu --set full --clock-control none --import-source on -k "regex:k_bnd_sym|k_response" -s 20 -c 2 -o gpurun_out/r01_sym_full -f python bench.py --steps 4 --warmup 30 --no-e2e --no-cpu-baseline --mode sym > gpurun_out/ncu_sym.log 2>&1
tail -2 gpurun_out/ncu_sym.log
timeout 600 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none -s 300 -c 60 --csv --log-file gpurun_out/r01_launches_sym.csv python bench.py --steps 20 --warmup 30 --no-e2e --no-cpu-baseline --mode sym > gpurun_out/ncu_sym_list.log 2>&1
python scripts/ncu_summarize.py gpurun_out/r01_launches_sym.csv

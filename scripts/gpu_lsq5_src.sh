mkdir -p gpurun_out
timeout 900 ncu --set full --clock-control none --import-source on --warp-sampling-interval 0 -k "regex:k_lsq_warp" -s 2 -c 1 -o gpurun_out/lsq5 -f python bench.py --steps 4 --warmup 5 --reps 1 --no-e2e --no-cpu-baseline --no-profile > gpurun_out/lsq5.log 2>&1
ncu -i gpurun_out/lsq5.ncu-rep --page source --csv --print-source cuda,sass -k regex:k_lsq > gpurun_out/lsq5_cs.csv 2>/dev/null
python scripts/ncu_cuda_lines.py gpurun_out/lsq5_cs.csv 30 > gpurun_out/lsq5_lines.txt 2>&1
python scripts/ncu_details.py gpurun_out/lsq5.ncu-rep k_lsq > gpurun_out/lsq5_details.txt 2>&1
rm -f gpurun_out/*.ncu-rep gpurun_out/lsq5_cs.csv

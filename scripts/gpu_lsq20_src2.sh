mkdir -p gpurun_out
timeout 900 ncu --set full --clock-control none --import-source on --warp-sampling-interval 0 -k "regex:k_lsq" -s 10 -c 1 -o gpurun_out/lsq20 -f python bench.py --config C3 --steps 4 --warmup 5 --reps 1 --no-e2e --no-cpu-baseline --no-profile > gpurun_out/lsq20.log 2>&1
ncu -i gpurun_out/lsq20.ncu-rep --page source --csv --print-source cuda,sass -k regex:k_lsq > gpurun_out/lsq20_cs.csv 2>&1
ncu -i gpurun_out/lsq20.ncu-rep --page source --csv --print-source cuda -k regex:k_lsq > gpurun_out/lsq20_c.csv 2>&1
head -c 3000 gpurun_out/lsq20_cs.csv > gpurun_out/lsq20_cs_head.txt
head -c 3000 gpurun_out/lsq20_c.csv > gpurun_out/lsq20_c_head.txt
ls -la gpurun_out/lsq20_c*.csv
rm -f gpurun_out/*.ncu-rep

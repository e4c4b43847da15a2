mkdir -p gpurun_out
timeout 900 ncu --set full --clock-control none --import-source on --warp-sampling-interval 0 -k "regex:k_lsq" -s 10 -c 1 -o gpurun_out/lsq20 -f python bench.py --config C3 --steps 4 --warmup 5 --reps 1 --no-e2e --no-cpu-baseline --no-profile > gpurun_out/lsq20.log 2>&1
python scripts/ncu_details.py gpurun_out/lsq20.ncu-rep k_lsq > gpurun_out/lsq20_details.txt 2>&1
ncu -i gpurun_out/lsq20.ncu-rep --page source --csv -k regex:k_lsq > gpurun_out/lsq20_src.csv 2>/dev/null
python scripts/ncu_srclines.py gpurun_out/lsq20_src.csv 40 > gpurun_out/lsq20_srctop.txt 2>&1
rm -f gpurun_out/*.ncu-rep

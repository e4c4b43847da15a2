mkdir -p gpurun_out
timeout 900 ncu --set full --clock-control none --import-source on --warp-sampling-interval 0 -k "regex:k_steps_fill" -s 10 -c 1 -o gpurun_out/f3t_full -f python bench.py --rule full --steps 4 --warmup 5 --reps 1 --no-e2e --no-cpu-baseline --no-profile > gpurun_out/f3t.log 2>&1
ncu -i gpurun_out/f3t_full.ncu-rep --page source --csv -k regex:k_steps_fill > gpurun_out/f3t_src.csv 2>/dev/null
python scripts/ncu_srclines.py gpurun_out/f3t_src.csv 45 > gpurun_out/f3t_srctop.txt 2>&1
rm -f gpurun_out/*.ncu-rep

mkdir -p gpurun_out
timeout 900 ncu --set full --clock-control none --import-source on --warp-sampling-interval 0 -k "regex:k_dst_inv|k_tridiag_reg" -s 20 -c 2 -o gpurun_out/tail -f python bench.py --steps 4 --warmup 10 --reps 1 --no-e2e --no-cpu-baseline --no-profile > gpurun_out/tail.log 2>&1
for k in k_dst_inv k_tridiag_reg; do
ncu -i gpurun_out/tail.ncu-rep --page source --csv --print-source cuda,sass -k regex:$k > gpurun_out/tail_cs_$k.csv 2>/dev/null
python scripts/ncu_cuda_lines.py gpurun_out/tail_cs_$k.csv 25 > gpurun_out/tail_lines_$k.txt 2>&1
done
rm -f gpurun_out/*.ncu-rep gpurun_out/tail_cs_*.csv

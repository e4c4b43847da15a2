mkdir -p gpurun_out
timeout 900 ncu --set full --clock-control none --import-source on --warp-sampling-interval 0 -k "regex:k_dst_inv|k_tridiag_reg|k_bnd_reduce" -s 30 -c 3 -o gpurun_out/tail -f python bench.py --steps 4 --warmup 10 --reps 1 --no-e2e --no-cpu-baseline --no-profile > gpurun_out/tail.log 2>&1
for k in k_dst_inv k_tridiag_reg k_bnd_reduce; do
python scripts/ncu_details.py gpurun_out/tail.ncu-rep $k > gpurun_out/tail_$k.txt 2>&1
ncu -i gpurun_out/tail.ncu-rep --page source --csv -k regex:$k > gpurun_out/tail_src_$k.csv 2>/dev/null
python scripts/ncu_srclines.py gpurun_out/tail_src_$k.csv 30 > gpurun_out/tail_srctop_$k.txt 2>&1
done
rm -f gpurun_out/*.ncu-rep gpurun_out/tail_src_*.csv

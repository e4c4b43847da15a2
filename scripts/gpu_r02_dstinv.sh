mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()"
timeout 900 ncu --set full --clock-control none --import-source on --warp-sampling-interval 0 -k "regex:k_dst_inv|k_tridiag_reg|k_lsq_warp" -s 30 -c 3 -o gpurun_out/r02_di -f python bench.py --steps 4 --warmup 30 --reps 1 --no-e2e --no-cpu-baseline --no-profile > gpurun_out/r02_di.log 2>&1
for k in k_dst_inv k_tridiag_reg k_lsq_warp; do
  ncu -i gpurun_out/r02_di.ncu-rep --page source --csv --print-source cuda -k regex:$k > gpurun_out/r02_di_cuda_$k.csv 2>/dev/null
  python scripts/ncu_details.py gpurun_out/r02_di.ncu-rep $k > gpurun_out/r02_di_$k.txt 2>&1
done
ls -la gpurun_out/r02_di_*
rm -f gpurun_out/*.ncu-rep

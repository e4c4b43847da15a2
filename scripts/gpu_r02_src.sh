mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()"
timeout 900 ncu --set full --clock-control none --import-source on --warp-sampling-interval 0 -k "regex:k_lsq_warp|k_tridiag_reg|k_current_from" -s 30 -c 3 -o gpurun_out/r02_src -f python bench.py --steps 4 --warmup 30 --reps 1 --no-e2e --no-cpu-baseline --no-profile > gpurun_out/r02_src.log 2>&1
tail -1 gpurun_out/r02_src.log
for k in k_lsq_warp k_tridiag_reg k_current_from; do ncu -i gpurun_out/r02_src.ncu-rep --page source --csv -k regex:$k > gpurun_out/r02_src_$k.csv 2>/dev/null; python scripts/ncu_srclines.py gpurun_out/r02_src_$k.csv 25 > gpurun_out/r02_srctop_$k.txt; done
rm -f gpurun_out/*.ncu-rep gpurun_out/r02_src_*.csv

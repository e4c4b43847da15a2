# round-2: launch list of the default bench + full captures of the latency-bound chain kernels
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()"
timeout 600 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none -s 400 -c 60 --csv --log-file gpurun_out/r02_launches_a.csv python bench.py --steps 20 --warmup 40 --reps 1 --no-e2e --no-cpu-baseline --no-profile > gpurun_out/r02_list.log 2>&1
python scripts/ncu_summarize.py gpurun_out/r02_launches_a.csv
timeout 900 ncu --set full --clock-control none --import-source on -k "regex:k_dst_inv|k_tridiag|k_lsq|k_bnd_reduce|k_resp_reduce|k_current|k_lr_mac|k_lr_fft|k_dst_fwd|k_sym_edge" -s 60 -c 10 -o gpurun_out/r02_tail -f python bench.py --steps 4 --warmup 30 --reps 1 --no-e2e --no-cpu-baseline --no-profile > gpurun_out/r02_tail.log 2>&1
tail -2 gpurun_out/r02_tail.log
for k in k_dst_inv k_tridiag k_lsq k_bnd_reduce k_resp_reduce k_current; do python scripts/ncu_details.py gpurun_out/r02_tail.ncu-rep $k > gpurun_out/r02_tail_$k.txt 2>&1; done
ncu -i gpurun_out/r02_tail.ncu-rep --page source --csv -k regex:k_dst_inv > gpurun_out/r02_src_dst_inv.csv 2>/dev/null
rm -f gpurun_out/*.ncu-rep

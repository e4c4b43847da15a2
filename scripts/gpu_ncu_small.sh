mkdir -p gpurun_out
timeout 900 ncu --set full --clock-control none --import-source on -k "regex:k_lsq|k_dst_fwd|k_dst_inv|k_normalize|k_basis" -s 20 -c 5 -o gpurun_out/prof_small -f python bench.py --steps 6 --warmup 5 --no-e2e --no-cpu-baseline > gpurun_out/ncu_small.log 2>&1
tail -1 gpurun_out/ncu_small.log

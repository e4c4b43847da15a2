mkdir -p gpurun_out
timeout 900 ncu --set full --cache-control none --clock-control none --import-source on -k "regex:k_lsq|k_dst_fwd|k_dst_inv|k_normalize|k_tridiag|k_response|k_lr_mac" -s 40 -c 7 -o gpurun_out/prof_small2 -f python bench.py --steps 6 --warmup 8 --no-e2e --no-cpu-baseline > gpurun_out/ncu_small.log 2>&1
tail -1 gpurun_out/ncu_small.log

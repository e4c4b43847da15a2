mkdir -p gpurun_out
timeout 900 ncu --set full --cache-control none --clock-control none --import-source on -k "regex:k_dst_fwd|k_dst_inv|k_tridiag|k_bnd_reduce" -s 20 -c 4 -o gpurun_out/prof_solve -f python bench.py --steps 6 --warmup 8 --no-e2e --no-cpu-baseline > gpurun_out/ncu_solve.log 2>&1
tail -1 gpurun_out/ncu_solve.log

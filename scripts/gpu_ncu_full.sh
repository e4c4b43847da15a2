mkdir -p gpurun_out
timeout 900 ncu --set full --clock-control none --import-source on -k "regex:k_response|k_bnd_lr|k_dst|k_tridiag|k_normalize|k_lsq|k_basis|k_current" -s 30 -c 9 -o gpurun_out/prof_full2 -f python bench.py --steps 6 --warmup 5 --no-e2e --no-cpu-baseline > gpurun_out/ncu_full.log 2>&1
tail -2 gpurun_out/ncu_full.log

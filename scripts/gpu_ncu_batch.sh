# ncu --set full of the batched tensor-core kernels (S = 4 slices, C4)
mkdir -p gpurun_out
timeout 900 ncu --set full --clock-control none --import-source on -k "regex:k_response_mma|k_bnd_tb_mma" -s 4 -c 2 -o gpurun_out/r01_batch_full -f python bench.py --steps 4 --warmup 4 --slices 4 > gpurun_out/ncu_batch.log 2>&1
tail -2 gpurun_out/ncu_batch.log

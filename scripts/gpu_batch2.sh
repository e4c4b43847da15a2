# batch tests + bench S = 4 (+ launch list of the two shared kernels)
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_batch.py -x -q 2>&1 | tail -2
for S in 4 8; do
  timeout 300 python bench.py --steps 400 --warmup 10 --slices $S > gpurun_out/bench_s$S.log 2>&1
  tail -1 gpurun_out/bench_s$S.log | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('S=$S', d['value'], d['ms_per_step'], d['roofline']['achieved'], d['roofline']['frac'], d['e2e']['value'])" || tail -5 gpurun_out/bench_s$S.log
done
timeout 600 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none -k "regex:mma" -s 4 -c 4 --csv --log-file gpurun_out/r01_launches_mma.csv python bench.py --steps 10 --warmup 10 --slices 4 > gpurun_out/ncu_s4.log 2>&1
python scripts/ncu_summarize.py gpurun_out/r01_launches_mma.csv

# k_response_mma variants at S = 4 (bench slice it/s + ncu duration), and the default bench line (sym mode)
mkdir -p gpurun_out
for L in paper_conf_sc_anteparawkbml23_b200/libefit_b200.so tune/libefit_*.so; do
  EFIT_B200_LIB=$PWD/$L timeout 300 python bench.py --steps 400 --warmup 10 --slices 4 2>&1 | tail -1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('$L', d['value'], d['ms_per_step'])" || echo "$L failed"
done
timeout 300 python bench.py 2>&1 | tail -1 > gpurun_out/bench_default.json
cat gpurun_out/bench_default.json | cut -c1-1500

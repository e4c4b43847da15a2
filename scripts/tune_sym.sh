# time the sym-mode fit step with each tuning variant in tune/, plus a parity spot check per variant
mkdir -p gpurun_out
for L in paper_conf_sc_anteparawkbml23_b200/libefit_b200.so tune/libefit_*.so; do
  EFIT_B200_LIB=$PWD/$L timeout 300 python -m pytest tests/test_gpu_parity.py -q -x -k "test_boundary_flux and 2-True" 2>&1 | tail -1
  EFIT_B200_LIB=$PWD/$L timeout 300 python bench.py --steps 1000 --warmup 20 --no-cpu-baseline --no-e2e --mode sym 2>&1 | tail -1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('$L', d['value'], d['config']['step_breakdown_us']['bnd_tb'], d['roofline']['achieved'])" || echo "$L failed"
done

# left/right path A/B per grid size: FFT chain (default) vs direct Toeplitz kernel (EFIT_LR_DIRECT=1)
mkdir -p gpurun_out
for c in C1 C2 C3 C4; do
for d in 0 1; do
if [ $d = 1 ]; then export EFIT_LR_DIRECT=1; else unset EFIT_LR_DIRECT; fi
timeout 300 python bench.py --config $c --steps 1000 --warmup 10 --no-cpu-baseline --no-e2e 2>&1 | tail -1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('$c direct=$d', d['value'], d['config']['step_breakdown_us'])" || echo "$c $d failed"
done
done

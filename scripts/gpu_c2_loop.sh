mkdir -p gpurun_out
for m in sym table; do MODE=$m timeout 300 python scripts/measure_c2_loop.py 2>&1 | tail -1; done
CFG=C4 MODE=sym timeout 300 python scripts/measure_c2_loop.py 2>&1 | tail -1

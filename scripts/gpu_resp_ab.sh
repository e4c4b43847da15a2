# single-slice response: fused basis (default) vs separate k_basis (EFIT_RESP_NOFUSE=1); GPU tests first
mkdir -p gpurun_out
timeout 900 python -m pytest tests -m gpu -x -q 2>&1 | tail -2
run() { timeout 300 python bench.py --steps 1000 --warmup 20 --no-cpu-baseline --no-e2e --mode $2 2>&1 | tail -1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); b=d['config']['step_breakdown_us']; print('$1 $2', d['value'], b['step'], b['response'], b['bnd_tb'], b['tail'], d['response_boundary']['frac'])" || echo "$1 failed"; }
run fused sym
EFIT_RESP_NOFUSE=1 run sep sym
run fused table
EFIT_RESP_NOFUSE=1 run sep table

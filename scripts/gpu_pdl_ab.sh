for r in 1 2; do
for v in 0 1; do if [ $v = 1 ]; then export EFIT_NO_PDL=1; else unset EFIT_NO_PDL; fi; timeout 300 python bench.py --steps 3000 --warmup 50 --no-e2e --no-cpu-baseline 2>&1 | python -c "import json,sys; d=json.loads(sys.stdin.readlines()[-1]); print('NO_PDL=$v', d['value'], d['config']['step_breakdown_us'])"; done
done

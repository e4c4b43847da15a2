# A/B of the staged k_tridiag_reg: GPU tests (solve parity), C4 bench, launch list of the tail
mkdir -p gpurun_out
timeout 1200 python -m pytest tests -m gpu -x -q 2>&1 | tail -3
for r in 1 2; do timeout 300 python bench.py --steps 1000 --no-cpu-baseline --no-e2e 2>&1 | tail -1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); print(d['value'], d['config']['step_breakdown_us'])"; done
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -s 300 -c 45 --csv --log-file gpurun_out/tailab.csv python bench.py --steps 20 --warmup 30 --reps 1 --no-e2e --no-cpu-baseline --no-profile > /dev/null 2>&1
python scripts/ncu_summarize.py gpurun_out/tailab.csv | grep -E 'tridiag|dst_inv|bnd_reduce|sum'

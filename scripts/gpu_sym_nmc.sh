# SYM-mode m-chunk sweep (EFIT_SYM_NMC): tail imbalance of 2080 tiles over 296 CTA slots
mkdir -p gpurun_out
for n in 1 2 3 4 5; do
  EFIT_SYM_NMC=$n timeout 300 python bench.py --steps 500 --warmup 20 --no-cpu-baseline --no-e2e --mode sym > gpurun_out/sym_nmc$n.log 2>&1
  echo -n "nmc=$n "; tail -1 gpurun_out/sym_nmc$n.log | python -c "import json,sys; d=json.loads(sys.stdin.read()); print(d['value'], d['config'].get('step_breakdown_us'), d['roofline']['achieved'], d['roofline']['frac'])"
done

# k_response chunk-size sweep at C4 (waves of CTAs vs per-CTA prologue)
for g in 0 256 384 512 640 1152; do
  if [ $g = 0 ]; then unset EFIT_RESP_GC; else export EFIT_RESP_GC=$g; fi
  timeout 300 python bench.py --steps 1000 --no-cpu-baseline --no-e2e > gpurun_out/respgc_$g.json 2>&1
  tail -1 gpurun_out/respgc_$g.json | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('gc', $g, d['value'], d['config']['step_breakdown_us']['response'])"
done

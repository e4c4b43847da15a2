# quick iteration: selected GPU tests ($TESTK), one bench mode ($MODE), ncu full capture of $NCUK
mkdir -p gpurun_out
timeout 900 python -m pytest tests -m gpu -x -q ${TESTK:+-k "$TESTK"} 2>&1 | tail -5
for m in ${MODES:-sym}; do
  timeout 300 python bench.py --steps 1000 --warmup 20 --no-cpu-baseline --no-e2e --mode $m > gpurun_out/bench_$m.log 2>&1
  tail -1 gpurun_out/bench_$m.log | python -c "import json,sys; d=json.loads(sys.stdin.read()); print(d['config']['green_mode'], d['value'], d['config']['step_breakdown_us'], d['roofline']['achieved'], d['roofline']['frac'])" || tail -5 gpurun_out/bench_$m.log
done
if [ -n "$NCUK" ]; then
  timeout 600 ncu --set full --clock-control none --import-source on -k "regex:$NCUK" -s 20 -c ${NCUC:-1} -o gpurun_out/${NCUO:-iter_full} python bench.py --steps 4 --warmup 30 --no-e2e --no-cpu-baseline --mode ${NCUMODE:-sym} > gpurun_out/ncu_iter.log 2>&1
  tail -1 gpurun_out/ncu_iter.log
fi

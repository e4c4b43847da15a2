timeout 900 python -m pytest tests -m gpu -x -q 2>&1 | tail -3
for cfg in C3 C4; do
  timeout 600 python bench.py --config $cfg --steps 1000 --warmup 20 --no-cpu-baseline --no-e2e 2>&1 | tail -1 | python -c "
import json,sys; d=json.loads(sys.stdin.read()); r=d['roofline']; rb=d['response_boundary']
print('$cfg', d['value'], 'it/s', d['ms_per_step'],'ms', 'tb_frac', r['frac'], 'rb_frac', rb and rb['frac'], 'init_s', d['config']['init_s'], d['config']['step_breakdown_us'])"
done
timeout 900 python bench.py --config C4 --mode otf --steps 30 --warmup 3 --no-cpu-baseline --no-e2e 2>&1 | tail -1 | python -c "
import json,sys; d=json.loads(sys.stdin.read());
print('C4 otf', d['value'], 'it/s', d['ms_per_step'],'ms', d['config']['step_breakdown_us'])"

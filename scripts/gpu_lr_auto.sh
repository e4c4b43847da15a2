# automatic left/right path choice: full GPU tests + C1..C4 bench
mkdir -p gpurun_out
timeout 900 python -m pytest tests -m gpu -x -q 2>&1 | tail -2
timeout 300 python __graft_entry__.py --smoke 2>&1 | tail -1
for c in C1 C2 C3 C4; do
timeout 300 python bench.py --config $c --steps 1000 --warmup 10 --no-cpu-baseline --no-e2e 2>&1 | tail -1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('$c', d['value'])" || echo "$c failed"
done
timeout 300 python bench.py --config C1 --slices 4 --steps 300 --warmup 5 2>&1 | tail -1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('C1 S=4', d['value'])" || echo "C1 batch failed"

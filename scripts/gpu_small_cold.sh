# C1-C3 bench lines with the cold-L2 value (tables fit in L2) and the L2-warm number beside it
mkdir -p gpurun_out
for c in C1 C2 C3; do for m in sym vh; do
  timeout 300 python bench.py --config $c --mode $m --steps 2000 --no-cpu-baseline --no-e2e > gpurun_out/r02b_bench_${c}_$m.json 2>&1
done; done
timeout 300 python bench.py --config C2 --rule full --steps 1000 --no-cpu-baseline --no-e2e > gpurun_out/r02b_bench_C2_f3.json 2>&1

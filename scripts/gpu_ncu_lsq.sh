# one full ncu capture of k_lsq<20> (C3 step) with source correlation; exports only (the report is large)
mkdir -p gpurun_out
timeout 600 ncu --set full --clock-control none --import-source on --warp-sampling-interval 0 -k "regex:k_lsq" -s 5 -c 1 -o /tmp/prof_lsq -f python bench.py --config C3 --steps 10 --warmup 10 --no-e2e --no-cpu-baseline > gpurun_out/ncu_lsq.log 2>&1
ncu -i /tmp/prof_lsq.ncu-rep --page source --csv --print-source sass > gpurun_out/lsq_sass.csv 2>&1
ncu -i /tmp/prof_lsq.ncu-rep --page source --csv --print-source cuda,sass > gpurun_out/lsq_cs.csv 2>&1
ls -la gpurun_out
python scripts/ncu_sass_lines.py gpurun_out/lsq_sass.csv gpurun_out/lsq_cs.csv 30

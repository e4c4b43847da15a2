# f3 (full steps_) measurement: bench lines (C4 diverted / limited, C2, C5), loop under the full rule,
# ncu launch list of the f3 step
mkdir -p gpurun_out
B="timeout 900 python bench.py --no-cpu-baseline"
$B --rule full --steps 500 > gpurun_out/f3_bench_c4_div.json 2> gpurun_out/f3_bench_c4_div.err; tail -1 gpurun_out/f3_bench_c4_div.json; tail -3 gpurun_out/f3_bench_c4_div.err
$B --rule full --shape limited --no-e2e --steps 500 > gpurun_out/f3_bench_c4_lim.json 2>&1; tail -1 gpurun_out/f3_bench_c4_lim.json
$B --rule full --config C2 --steps 2000 > gpurun_out/f3_bench_c2_div.json 2>&1; tail -1 gpurun_out/f3_bench_c2_div.json
$B --rule full --config C5 --steps 200 > gpurun_out/f3_bench_c5_div.json 2>&1; tail -1 gpurun_out/f3_bench_c5_div.json
timeout 600 python bench.py --loop --rule full --config C2 --steps 400 > gpurun_out/f3_loop_c2.json 2>&1; tail -c 600 gpurun_out/f3_loop_c2.json
timeout 900 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none -s 300 -c 48 --csv --log-file gpurun_out/f3_launches_c4.csv python bench.py --rule full --steps 20 --warmup 30 --reps 1 --no-e2e --no-cpu-baseline --no-profile > gpurun_out/f3_ncu_list.log 2>&1
python scripts/ncu_summarize.py gpurun_out/f3_launches_c4.csv > gpurun_out/f3_launches_c4_summary.txt 2>&1; cat gpurun_out/f3_launches_c4_summary.txt | head -30

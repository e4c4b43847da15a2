# Round-2 (second session) evidence run on one B200: all GPU tests, smoke, the default bench line,
# every config/mode, the f3 steps_ rule, loops, the batch, the launch list and full ncu captures.
set -x
mkdir -p gpurun_out
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,memory.total --format=csv
timeout 1500 python -m pytest tests -m gpu -q 2>&1 | tail -5 > gpurun_out/r02b_final_gputests.txt
timeout 300 python __graft_entry__.py --smoke 2>&1 | tail -2 > gpurun_out/r02b_final_smoke.txt
B="timeout 900 python bench.py --no-cpu-baseline"
timeout 900 python bench.py > gpurun_out/r02b_bench_c4_sym.json 2>gpurun_out/r02b_bench_c4_sym.err
for m in table vh otf-sym; do $B --no-e2e --mode $m --steps 500 > gpurun_out/r02b_bench_c4_$m.json 2>&1; done
for c in C1 C2 C3; do $B --no-e2e --config $c --steps 2000 > gpurun_out/r02b_bench_${c}_sym.json 2>&1; done
for c in C1 C2 C3; do $B --no-e2e --config $c --mode vh --steps 2000 > gpurun_out/r02b_bench_${c}_vh.json 2>&1; done
for m in sym vh table; do $B --no-e2e --config C5 --mode $m --steps 200 > gpurun_out/r02b_bench_c5_$m.json 2>&1; done
for c in C2 C4 C5; do $B --no-e2e --rule full --config $c --steps 300 > gpurun_out/r02b_bench_${c}_f3.json 2>&1; done
$B --no-e2e --rule full --shape limited --steps 500 > gpurun_out/r02b_bench_c4_f3_limited.json 2>&1
for S in 4 8; do $B --slices $S --steps 500 > gpurun_out/r02b_bench_c4_s$S.json 2>&1; done
timeout 600 python bench.py --loop --config C2 --steps 400 > gpurun_out/r02b_loop_C2.json 2>&1
timeout 900 python bench.py --loop --config C4 --steps 400 > gpurun_out/r02b_loop_C4.json 2>&1
timeout 600 python bench.py --loop --config C2 --rule full --steps 400 > gpurun_out/r02b_loop_C2_f3.json 2>&1
timeout 300 python bench.py --impl reference --steps 2 --warmup 1 > gpurun_out/r02b_bench_reference.json 2>&1
timeout 900 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none -s 300 -c 45 --csv --log-file gpurun_out/r02b_launches_c4_sym.csv python bench.py --steps 20 --warmup 30 --reps 1 --no-e2e --no-cpu-baseline --no-profile > gpurun_out/r02b_ncu_list.log 2>&1
python scripts/ncu_summarize.py gpurun_out/r02b_launches_c4_sym.csv > gpurun_out/r02b_launches_c4_sym_summary.txt 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k "regex:k_bnd_sym|k_response" -s 20 -c 2 -o gpurun_out/r02b_full -f python bench.py --steps 4 --warmup 30 --reps 1 --no-e2e --no-cpu-baseline --no-profile > gpurun_out/r02b_ncu_full.log 2>&1
python scripts/ncu_details.py gpurun_out/r02b_full.ncu-rep k_bnd_sym > gpurun_out/r02b_full_sym.txt 2>&1
python scripts/ncu_details.py gpurun_out/r02b_full.ncu-rep k_response > gpurun_out/r02b_full_resp.txt 2>&1
rm -f gpurun_out/*.ncu-rep

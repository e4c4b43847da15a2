# Round-2 evidence run (one B200): benches of every config/mode, the full loop, the batch, the
# launch list and full ncu captures of the dominant kernels.  Results -> gpurun_out/r02_*.
set -x
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()"
B="timeout 900 python bench.py --no-cpu-baseline"
$B > gpurun_out/r02_bench_c4_sym.json 2>gpurun_out/r02_bench_c4_sym.err
for m in table vh otf-sym; do $B --no-e2e --mode $m --steps 500 > gpurun_out/r02_bench_c4_$m.json 2>&1; done
for c in C1 C2 C3; do $B --no-e2e --config $c --steps 2000 > gpurun_out/r02_bench_${c}_sym.json 2>&1; done
for c in C1 C2 C3; do $B --no-e2e --config $c --mode vh --steps 2000 > gpurun_out/r02_bench_${c}_vh.json 2>&1; done
for m in sym vh table; do $B --no-e2e --config C5 --mode $m --steps 200 > gpurun_out/r02_bench_c5_$m.json 2>&1; done
for S in 4 8; do $B --slices $S --steps 500 > gpurun_out/r02_bench_c4_s$S.json 2>&1; done
timeout 600 python bench.py --loop --config C2 --steps 400 > gpurun_out/r02_loop_c2.json 2>&1
timeout 900 python bench.py --loop --config C4 --steps 400 > gpurun_out/r02_loop_c4.json 2>&1
timeout 600 python bench.py --loop --config C2 --mode vh --steps 400 > gpurun_out/r02_loop_c2_vh.json 2>&1
timeout 900 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none -s 300 -c 45 --csv --log-file gpurun_out/r02_launches_c4_sym.csv python bench.py --steps 20 --warmup 30 --reps 1 --no-e2e --no-cpu-baseline --no-profile > gpurun_out/r02_ncu_list.log 2>&1
python scripts/ncu_summarize.py gpurun_out/r02_launches_c4_sym.csv > gpurun_out/r02_launches_c4_sym_summary.txt
timeout 900 ncu --set full --clock-control none --import-source on -k "regex:k_bnd_sym|k_response|k_bnd_tb<" -s 20 -c 3 -o gpurun_out/r02_full -f python bench.py --steps 4 --warmup 30 --reps 1 --no-e2e --no-cpu-baseline --no-profile > gpurun_out/r02_ncu_full.log 2>&1
python scripts/ncu_to_summary.py gpurun_out/r02_full.ncu-rep "default sym mode" k_bnd_sym k_response > gpurun_out/r02_ncu_summary_update.txt 2>&1
python scripts/ncu_details.py gpurun_out/r02_full.ncu-rep k_bnd_sym > gpurun_out/r02_full_sym.txt 2>&1
python scripts/ncu_details.py gpurun_out/r02_full.ncu-rep k_response > gpurun_out/r02_full_resp.txt 2>&1
cp profiles/ncu_summary.json gpurun_out/r02_ncu_summary.json
rm -f gpurun_out/*.ncu-rep

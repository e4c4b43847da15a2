# round-1 final evidence: launch list of the default bench (sym), full capture of the two streams,
# FP64 instruction counts of the on-the-fly kernels (ALU roofline)
mkdir -p gpurun_out
timeout 600 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none -s 300 -c 45 --csv --log-file gpurun_out/r01_launches_final.csv python bench.py --steps 20 --warmup 30 --no-e2e --no-cpu-baseline > gpurun_out/ncu_final_list.log 2>&1
python scripts/ncu_summarize.py gpurun_out/r01_launches_final.csv
timeout 900 ncu --set full --clock-control none --import-source on -k "regex:k_bnd_sym|k_response" -s 20 -c 2 -o gpurun_out/r01_final_full -f python bench.py --steps 4 --warmup 30 --no-e2e --no-cpu-baseline > gpurun_out/ncu_final_full.log 2>&1
tail -1 gpurun_out/ncu_final_full.log
for m in otf otf-sym; do
timeout 600 ncu --metrics gpu__time_duration.sum,smsp__sass_thread_inst_executed_op_dadd_pred_on.sum,smsp__sass_thread_inst_executed_op_dmul_pred_on.sum,smsp__sass_thread_inst_executed_op_dfma_pred_on.sum,sm__pipe_fp64_cycles_active.avg.pct_of_peak_sustained_active --clock-control none -k "regex:k_bnd_tb_otf|k_bnd_sym" -s 2 -c 2 --csv --log-file gpurun_out/r01_otf_$m.csv python bench.py --steps 3 --warmup 3 --no-e2e --no-cpu-baseline --mode $m > gpurun_out/ncu_otf_$m.log 2>&1
python -c "import csv,sys; r=list(csv.reader(open(\"gpurun_out/r01_otf_$m.csv\"))); i=[k for k,l in enumerate(r) if l and l[0]==\"ID\"][0]; h=r[i]; [print(x[h.index(\"Kernel Name\")][:22], x[h.index(\"Metric Name\")], x[h.index(\"Metric Value\")]) for x in r[i+1:i+11]]"
done
# keep gpurun_out small (<= 64 MiB comes back): export the full capture as CSV and drop the report
ncu -i gpurun_out/r01_final_full.ncu-rep --page raw --csv > gpurun_out/r01_final_full_raw.csv 2>/dev/null
python scripts/ncu_details.py gpurun_out/r01_final_full.ncu-rep k_bnd_sym > gpurun_out/r01_final_full_sym.txt 2>&1
python scripts/ncu_details.py gpurun_out/r01_final_full.ncu-rep k_response > gpurun_out/r01_final_full_resp.txt 2>&1
rm -f gpurun_out/*.ncu-rep
du -sh gpurun_out

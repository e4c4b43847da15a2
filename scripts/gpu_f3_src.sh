# SASS-level stall sampling of the f3 one-CTA kernels (C4, diverted)
mkdir -p gpurun_out
timeout 900 ncu --set full --clock-control none --import-source on -k "regex:k_steps_f" -s 20 -c 2 -o gpurun_out/f3s_full -f python bench.py --rule full --steps 4 --warmup 10 --reps 1 --no-e2e --no-cpu-baseline --no-profile > gpurun_out/f3s_ncu_full.log 2>&1
for k in k_steps_final k_steps_fill; do
  ncu -i gpurun_out/f3s_full.ncu-rep --page source --csv -k regex:$k > gpurun_out/f3s_src_$k.csv 2>/dev/null
  python scripts/ncu_srclines.py gpurun_out/f3s_src_$k.csv 40 > gpurun_out/f3s_srctop_$k.txt 2>&1
done
rm -f gpurun_out/*.ncu-rep

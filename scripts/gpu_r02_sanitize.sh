mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()"
for tool in memcheck racecheck synccheck initcheck; do
  timeout 900 compute-sanitizer --tool $tool --print-limit 20 python scripts/sanitize_small.py 33 > gpurun_out/r02_sanitize_$tool.txt 2>&1
  echo "$tool rc=$?: $(tail -2 gpurun_out/r02_sanitize_$tool.txt | tr '\n' ' ')"
done

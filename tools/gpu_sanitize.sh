mkdir -p gpurun_out/san
for tool in memcheck initcheck synccheck racecheck; do
  timeout 1200 compute-sanitizer --tool $tool --print-limit 20 python tools/sanitize_run.py C1 > gpurun_out/san/$tool.log 2>&1
  echo "$tool rc=$?"; grep -E "ERROR SUMMARY|Invalid|Uninitialized|hazard" gpurun_out/san/$tool.log | head -5
done

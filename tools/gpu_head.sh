# HEAD check: GPU tests (incl. slow), smoke, bench line, sanitizer logs
mkdir -p gpurun_out/h
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv > gpurun_out/h/gpu.txt 2>&1
timeout 2400 python -m pytest tests -m gpu -q -rf --durations=15 > gpurun_out/h/gpu_tests.log 2>&1; echo "pytest rc=$?" >> gpurun_out/h/gpu_tests.log
tail -25 gpurun_out/h/gpu_tests.log
timeout 600 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/h/smoke.log 2>&1; echo "smoke rc=$?" >> gpurun_out/h/smoke.log
tail -2 gpurun_out/h/smoke.log
timeout 1500 python bench.py > gpurun_out/h/bench.json 2> gpurun_out/h/bench.err; echo "bench rc=$?"
tail -c 1500 gpurun_out/h/bench.err
mkdir -p gpurun_out/san
for tool in memcheck initcheck synccheck racecheck; do
  timeout 900 compute-sanitizer --tool $tool --print-limit 20 python tools/sanitize_run.py C1 > gpurun_out/san/$tool.log 2>&1
  echo "$tool rc=$?"; grep -E "ERROR SUMMARY|Invalid|Uninitialized|hazard" gpurun_out/san/$tool.log | head -5
done

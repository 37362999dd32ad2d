# full GPU test suite (incl. slow) + smoke
mkdir -p gpurun_out
timeout 2400 python -m pytest tests -m gpu -q -rf -x --durations=15 > gpurun_out/gpu_tests.log 2>&1; echo "pytest rc=$?" >> gpurun_out/gpu_tests.log
timeout 600 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke.log 2>&1; echo "smoke rc=$?" >> gpurun_out/smoke.log
tail -25 gpurun_out/gpu_tests.log; tail -3 gpurun_out/smoke.log

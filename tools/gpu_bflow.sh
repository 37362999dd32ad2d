mkdir -p gpurun_out/bf
timeout 420 python -m pytest tests/test_gpu_parity.py tests/test_gpu_backward_update.py -q -x -rf -k "not c4" > gpurun_out/bf/tests.log 2>&1; echo "tests rc=$?"; tail -3 gpurun_out/bf/tests.log
for m in 0 1; do
  INSTA_BWD_FLOW=$m timeout 300 python tools/sl_time.py C4 0 0 2>&1 | head -1
  INSTA_BWD_FLOW=$m timeout 300 python tools/sl_time.py C4 1 0 2>&1 | head -1
done

timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_incremental.py -x -q -m "gpu and not slow" 2>&1 | tail -3
for s in 0 3; do timeout 300 python tools/sl_time.py C4 0 $s 2>&1 | tail -2; done
timeout 300 python tools/sl_time.py C4 1 0 2>&1 | tail -2

timeout 1500 python -m pytest tests/test_gpu_parity.py tests/test_gpu_backward_update.py tests/test_gpu_incremental.py tests/test_gpu_size.py -q -x -rf 2>&1 | tail -2
for r in 1 2; do timeout 300 python tools/sl_time.py C4 0 0 2>&1 | head -1; done

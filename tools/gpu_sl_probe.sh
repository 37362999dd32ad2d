timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_incremental.py -q -m "gpu" -rf 2>&1 | grep -E "FAILED|passed|failed|Error" | head
timeout 300 python tools/sl_time.py C4 0 0 2>&1 | grep -E "C4|cone|update"

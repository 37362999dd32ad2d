INSTA_DEBUG_PLACE=1 timeout 900 python -m pytest tests/test_gpu_incremental.py tests/test_gpu_place.py -q -x -s -m gpu -k "c3_incremental or timing_loss" 2>&1 | grep -E "DBG|passed|failed" | tail -8

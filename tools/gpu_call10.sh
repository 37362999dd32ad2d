timeout 900 python -m pytest tests/test_gpu_topk.py -x -q -m "gpu and not slow" 2>&1 | tail -2
timeout 300 python tools/topk_bench.py C4 1 8 32 2>&1 | tail -3

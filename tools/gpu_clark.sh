timeout 600 python -m pytest tests/test_gpu_clark.py -q -x 2>&1 | tail -2
timeout 600 python tools/clark_bench.py C4 2>&1 | tail -3

timeout 900 python -m pytest tests/test_gpu_clark.py -x -q 2>&1 | tail -4
timeout 300 python tools/clark_bench.py C4 2>&1 | tail -2

timeout 600 python -m pytest tests/test_gpu_place.py -q -x 2>&1 | tail -3
timeout 900 python -m pytest tests/test_gpu_clark.py tests/test_gpu_place.py -q -x 2>&1 | tail -3
timeout 900 python -m pytest tests/test_gpu_next_edges.py tests/test_gpu_place.py -q -x 2>&1 | tail -3

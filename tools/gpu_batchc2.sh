timeout 900 python -m pytest tests/test_gpu_batch.py -q -x -rf -k "c2" 2>&1 | tail -3

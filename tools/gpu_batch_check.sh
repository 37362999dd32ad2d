# batched path: parity tests + steady-state timing (tools/batch_debug.py)
timeout 900 python -m pytest tests/test_gpu_batch.py -q -x 2>&1 | tail -1
DUMP_AFTER=300 timeout 300 python tools/batch_debug.py C4 2>&1 | tail -3

timeout 900 python -m pytest tests/test_gpu_parity.py -q -x -rf -k "unstaged or stage_folded or heavy_fanout or schedules" 2>&1 | tail -3

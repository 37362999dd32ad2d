timeout 900 python -m pytest tests/test_gpu_clark.py -x -q 2>&1 | tail -2
timeout 300 python tools/clark_bench.py C4 2>&1 | tail -1
timeout 300 ncu --metrics gpu__time_duration.sum --clock-control none -k regex:cl_bwd -s 324 -c 162 --csv --log-file gpurun_out/clark_levels.csv python tools/clark_bench.py C4 > /dev/null 2>&1; echo ncu=$?

timeout 900 python -m pytest tests/test_gpu_topk.py -x -q -m "gpu and not slow" 2>&1 | tail -2
timeout 300 python tools/topk_bench.py C4 8 32 2>&1 | tail -2
timeout 600 ncu --set full --import-source on --clock-control none -k regex:tk_level_kernel -s 60 -c 1 -o gpurun_out/prof_topk_multi2 -f python tools/topk_bench.py C4 32 > gpurun_out/ncu_topk3.log 2>&1; echo ncu_rc=$?

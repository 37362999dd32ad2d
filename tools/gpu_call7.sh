timeout 900 python -m pytest tests/test_gpu_topk.py -x -q -m "gpu and not slow" 2>&1 | tail -3
VARIANT=m4 timeout 300 python tools/topk_bench.py C4 1 8 32 2>&1 | tail -3
VARIANT=m3 INSTA_ROOT=$PWD/build_variants/m3 timeout 300 python tools/topk_bench.py C4 32 2>&1 | tail -1
VARIANT=m5 INSTA_ROOT=$PWD/build_variants/m5 timeout 300 python tools/topk_bench.py C4 32 2>&1 | tail -1
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -k regex:"tk_level|tk_one" -s 640 -c 320 --csv --log-file gpurun_out/topk_levels2.csv python tools/topk_bench.py C4 32 > /dev/null 2>&1; echo ncu_rc=$?

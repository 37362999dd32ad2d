INSTA_ROOT=$PWD/build_variants/stats timeout 300 python tools/topk_stats.py C4 32 2>&1 | tail -2
timeout 600 ncu --set full --import-source on --clock-control none -k regex:tk_level_kernel -s 60 -c 1 -o gpurun_out/prof_topk_multi -f python tools/topk_bench.py C4 32 > gpurun_out/ncu_topk2.log 2>&1; echo ncu_rc=$?

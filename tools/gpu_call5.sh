export DUMP_AFTER=100
for i in 1 2 3; do timeout 150 python tools/batch_debug.py 2>&1 | tail -3; FWD_FIRST=1 timeout 150 python tools/batch_debug.py 2>&1 | tail -2; done
timeout 600 python bench.py --steps 20 --warmup 5 > gpurun_out/bench.json 2> gpurun_out/bench.err; echo bench_rc=$?
cat gpurun_out/bench.json
timeout 600 ncu --set full --import-source on --clock-control none -k regex:tk_level_kernel -s 100 -c 1 -o gpurun_out/prof_topk -f python tools/topk_bench.py C4 32 > gpurun_out/ncu_topk.log 2>&1; echo ncu_rc=$?
tail -3 gpurun_out/ncu_topk.log

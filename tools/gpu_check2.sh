mkdir -p gpurun_out/c2
timeout 1200 python -m pytest tests/test_gpu_place.py tests/test_gpu_parity.py tests/test_gpu_incremental.py tests/test_gpu_size.py -q -x > gpurun_out/c2/tests.log 2>&1; echo "tests rc=$?" >> gpurun_out/c2/tests.log
tail -3 gpurun_out/c2/tests.log
for v in 0 1; do INSTA_BWD_PREFILL=$v timeout 300 python tools/sl_time.py C4 0 2>&1 | head -1; done > gpurun_out/c2/ab.log
for v in 0 1; do INSTA_BWD_PREFILL=$v timeout 300 python tools/sl_time.py C4 1 2>&1 | head -1; done >> gpurun_out/c2/ab.log
cat gpurun_out/c2/ab.log
timeout 900 python bench.py --steps 10 --warmup 3 --e2e-steps 0 --no-cpu-baseline --batch-scenarios 0 --topk 0 --clark 0 --cold 0 --incremental 0 > gpurun_out/c2/bench.json 2> gpurun_out/c2/bench.err; echo "bench rc=$?"

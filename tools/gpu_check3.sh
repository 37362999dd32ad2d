mkdir -p gpurun_out/c3
timeout 1200 python -m pytest tests/test_gpu_batch.py tests/test_gpu_incremental.py tests/test_gpu_place.py tests/test_gpu_size.py -q -x > gpurun_out/c3/tests.log 2>&1; echo "tests rc=$?" >> gpurun_out/c3/tests.log
tail -3 gpurun_out/c3/tests.log
timeout 600 python tools/cone_probe.py C4 1e-7 1e-6 1e-5 > gpurun_out/c3/cone_c4.log 2>&1; echo "cone rc=$?"
timeout 900 python bench.py --steps 10 --warmup 3 --e2e-steps 0 --no-cpu-baseline --topk 0 --clark 0 --cold 0 --lse 0 --place 0 > gpurun_out/c3/bench.json 2> gpurun_out/c3/bench.err; echo "bench rc=$?"

mkdir -p gpurun_out/bu
timeout 420 python -m pytest tests/test_gpu_backward_update.py tests/test_gpu_size.py tests/test_gpu_incremental.py -q -x -rf > gpurun_out/bu/tests.log 2>&1; echo "tests rc=$?"; tail -15 gpurun_out/bu/tests.log
timeout 600 python bench.py --steps 5 --warmup 3 --e2e-steps 0 --no-cpu-baseline --batch-scenarios 0 --topk 0 --topk-wide 0 --clark 0 --lse 0 --cold 0 --place 0 --c3-steps 10 > gpurun_out/bu/bench.json 2> gpurun_out/bu/bench.err; echo "bench rc=$?"; tail -c 300 gpurun_out/bu/bench.err
python -c "import json;d=json.load(open('gpurun_out/bu/bench.json'));print(json.dumps(d['incremental']['C4_backward_update'],indent=0))"

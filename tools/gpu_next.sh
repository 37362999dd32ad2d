mkdir -p gpurun_out/nx2
timeout 900 python -m pytest tests/test_gpu_topk.py tests/test_gpu_place.py -q -x -rf > gpurun_out/nx2/tests.log 2>&1; echo "tests rc=$?"; tail -3 gpurun_out/nx2/tests.log
timeout 1200 python bench.py --steps 3 --warmup 3 --e2e-steps 0 --no-cpu-baseline --batch-scenarios 0 --clark 0 --lse 0 --cold 0 --incremental 0 > gpurun_out/nx2/bench.json 2> gpurun_out/nx2/bench.err; echo "bench rc=$?"; tail -c 300 gpurun_out/nx2/bench.err
python -c "import json;d=json.load(open('gpurun_out/nx2/bench.json'));print(json.dumps(d['place']));print(json.dumps(d['topk']));print(json.dumps(d['topk_wide']))"

mkdir -p gpurun_out/ev
timeout 600 python -m pytest tests/test_gpu_batch.py -q -x -rf > gpurun_out/ev/tests.log 2>&1; echo "tests rc=$?"; tail -3 gpurun_out/ev/tests.log
timeout 900 python bench.py --steps 3 --warmup 3 --e2e-steps 0 --no-cpu-baseline --topk 0 --topk-wide 0 --clark 0 --lse 0 --cold 0 --place 0 --incremental 0 > gpurun_out/ev/bench.json 2> gpurun_out/ev/bench.err; echo "bench rc=$?"; tail -c 300 gpurun_out/ev/bench.err
python -c "import json;d=json.load(open('gpurun_out/ev/bench.json'));print(json.dumps(d['batched']))"

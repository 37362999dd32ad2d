mkdir -p gpurun_out/ct
cd build_variants/phx && timeout 300 python tools/cone_trace.py C3 ../../gpurun_out/ct > ../../gpurun_out/ct/c3.txt 2>&1; echo rc=$?
cd ../.. && head -80 gpurun_out/ct/c3.txt
timeout 600 python bench.py --steps 3 --warmup 3 --e2e-steps 0 --no-cpu-baseline --batch-scenarios 0 --topk 0 --topk-wide 0 --clark 0 --lse 0 --cold 0 --place 0 --c3-steps 20 > gpurun_out/ct/bench.json 2> gpurun_out/ct/bench.err; echo "bench rc=$?"
python -c "import json;d=json.load(open('gpurun_out/ct/bench.json'))['incremental'];print(json.dumps(d['C3_1pct_steps']));print(json.dumps(d['C4_small_updates']))"
timeout 600 python -m pytest tests/test_gpu_incremental.py tests/test_gpu_backward_update.py tests/test_gpu_batch.py -q -x 2>&1 | tail -2

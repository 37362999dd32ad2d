timeout 600 python -m pytest tests/test_gpu_incremental.py tests/test_gpu_parity.py -q -x 2>&1 | tail -2
timeout 600 python bench.py --steps 5 --warmup 3 --batch-scenarios 0 --topk 0 --clark 0 --no-cpu-baseline 2>&1 | python -c "import json,sys; d=json.loads(sys.stdin.read().strip().splitlines()[-1]); print(json.dumps(d['e2e'])); print(d['config']['tns'], d['ms_per_step'])"

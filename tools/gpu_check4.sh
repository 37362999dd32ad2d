mkdir -p gpurun_out/c4 /tmp/tr
INSTA_SL_TRACE=/tmp/tr timeout 600 python tools/eval_probe.py C4 512 > gpurun_out/c4/eval.log 2>&1; echo "eval rc=$?"
timeout 1500 python -m pytest tests/test_gpu_topk.py -q -x > gpurun_out/c4/topk.log 2>&1; echo "topk rc=$?" >> gpurun_out/c4/topk.log
tail -3 gpurun_out/c4/topk.log
timeout 900 python bench.py --steps 5 --warmup 3 --e2e-steps 0 --no-cpu-baseline --batch-scenarios 0 --clark 0 --cold 0 --lse 0 --place 0 --incremental 0 > gpurun_out/c4/bench.json 2> gpurun_out/c4/bench.err; echo "bench rc=$?"

# Quick GPU iteration (run under gpurun): parity subset, bench, optional trace.
mkdir -p gpurun_out
timeout 600 python -m pytest tests -m "gpu and not slow" -x -q ${TESTS:+-k "$TESTS"} > gpurun_out/gpu_tests.log 2>&1; echo tests_rc=$?
tail -3 gpurun_out/gpu_tests.log
INSTA_DEBUG=1 timeout 600 python bench.py --steps 20 --warmup 5 ${BENCH_ARGS:-} > gpurun_out/bench.json 2> gpurun_out/bench.err; echo bench_rc=$?
grep insta gpurun_out/bench.err | head -3
python -c "
import json; d=json.load(open('gpurun_out/bench.json'))
print('fwd_ms', d['fwd_ms'], 'bwd_ms', d['bwd_ms'], 'value', d['value'], 'frac', d['roofline']['frac'])
b=d.get('batched') or {}; print('batched evals/s', b.get('evals_per_s'))
"
if [ -n "$TRACE" ]; then SPREAD=${SPREAD:-20:30} timeout 600 python tools/trace_run.py C4 > gpurun_out/trace_c4.txt 2>&1; head -4 gpurun_out/trace_c4.txt; grep -A3 "bwd_trace.bin: grid" gpurun_out/trace_c4.txt | head -3; fi
if [ -n "$NCU" ]; then timeout 600 ncu --set full --clock-control none --import-source on -k regex:"$NCU" -s 2 -c 1 -o gpurun_out/prof_q -f python bench.py --steps 1 --warmup 3 --e2e-steps 0 --no-cpu-baseline --batch-scenarios 0 > gpurun_out/ncu_q.log 2>&1; echo ncu_rc=$?; fi

# quick GPU check (run under gpurun): build, a pytest selection ($TESTS), one bench run
set -x
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || tail -20 gpurun_out/build.log
timeout 900 python -m pytest tests -m gpu -q -x ${TESTS:-} > gpurun_out/gpu_tests.log 2>&1; echo tests_rc=$?
tail -15 gpurun_out/gpu_tests.log
if [ "${BENCH:-1}" = "1" ]; then
timeout 600 python bench.py ${BENCH_ARGS:-} > gpurun_out/bench.json 2> gpurun_out/bench.err; echo bench_rc=$?
cat gpurun_out/bench.json; tail -5 gpurun_out/bench.err
fi

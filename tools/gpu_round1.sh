# GPU session script (run under gpurun): build, tests, bench, ncu evidence.
set -x
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
timeout 600 python -m pytest tests -m "gpu and not slow" -q -x > gpurun_out/gpu_tests.log 2>&1; echo tests_rc=$?
tail -15 gpurun_out/gpu_tests.log
timeout 600 python bench.py --steps 20 --warmup 5 > gpurun_out/bench.json 2> gpurun_out/bench.err; echo bench_rc=$?
cat gpurun_out/bench.json; tail -5 gpurun_out/bench.err
if [ "${PROFILE:-1}" = "1" ]; then
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches.csv python bench.py --steps 2 --warmup 3 --e2e-steps 0 --no-cpu-baseline > gpurun_out/ncu_list.log 2>&1; echo ncu1_rc=$?
timeout 900 ncu --set full --clock-control none --import-source on -k regex:"fwd_kernel|bwdf_kernel" -s 6 -c 2 -o gpurun_out/prof_c4 -f python bench.py --steps 1 --warmup 3 --e2e-steps 0 --no-cpu-baseline > gpurun_out/ncu_full.log 2>&1; echo ncu2_rc=$?
tail -3 gpurun_out/ncu_full.log
fi
if [ "${SLOW:-1}" = "1" ]; then
timeout 900 python -m pytest tests -m "gpu and slow" -q > gpurun_out/gpu_slow.log 2>&1; echo slow_rc=$?
tail -15 gpurun_out/gpu_slow.log
fi

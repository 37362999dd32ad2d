# full check of HEAD: GPU tests, smoke, bench line, launch list, ncu of the default fwd/bwd
mkdir -p gpurun_out/f6
timeout 1800 python -m pytest tests -m gpu -q -rf --durations=8 > gpurun_out/f6/gpu_tests.log 2>&1; echo "pytest rc=$?" >> gpurun_out/f6/gpu_tests.log
tail -14 gpurun_out/f6/gpu_tests.log
timeout 600 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/f6/smoke.log 2>&1; echo "smoke rc=$?"; tail -1 gpurun_out/f6/smoke.log
timeout 1500 python bench.py > gpurun_out/f6/bench.json 2> gpurun_out/f6/bench.err; echo "bench rc=$?"
tail -c 400 gpurun_out/f6/bench.err
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/f6/launches.csv python bench.py --steps 2 --warmup 3 --e2e-steps 0 --no-cpu-baseline --batch-scenarios 0 --topk 0 --topk-wide 0 --clark 0 --lse 0 --cold 0 --incremental 0 --place 0 > /dev/null 2>&1; echo "ncu list rc=$?"
timeout 1200 ncu --set full --import-source on --clock-control none -k regex:"fwdx_kernel|bwdl_kernel|slack_kernel|bwd_prep" -s 8 -c 4 -o gpurun_out/f6/full_c4 python bench.py --steps 3 --warmup 3 --e2e-steps 0 --no-cpu-baseline --batch-scenarios 0 --topk 0 --topk-wide 0 --clark 0 --lse 0 --cold 0 --incremental 0 --place 0 > gpurun_out/f6/ncu_full.log 2>&1; echo "ncu full rc=$?"

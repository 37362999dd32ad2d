python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1; echo build=$?; tail -3 gpurun_out/build.log
timeout 900 python -m pytest tests/test_gpu_place.py tests/test_gpu_size.py tests/test_gpu_topk.py -q -x 2>&1 | grep -E "passed|failed|^E " | head -20

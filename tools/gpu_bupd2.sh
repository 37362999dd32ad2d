mkdir -p gpurun_out/bu2
timeout 420 python -m pytest tests/test_gpu_backward_update.py tests/test_gpu_size.py -q -x -rf > gpurun_out/bu2/tests.log 2>&1; echo "tests rc=$?"; tail -3 gpurun_out/bu2/tests.log

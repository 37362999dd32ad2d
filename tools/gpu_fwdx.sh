# entry-parallel forward: parity (schedule 3 + schedule 0 via INSTA_FWDX) and timing
mkdir -p gpurun_out/fx
for m in 1 2; do
  INSTA_FWDX=$m timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_incremental.py tests/test_gpu_next_edges.py -q -m gpu -x -k "not c4" > gpurun_out/fx/par_$m.log 2>&1; echo "parity m=$m rc=$?"; tail -3 gpurun_out/fx/par_$m.log
done
for m in 0 1 2; do
  INSTA_FWDX=$m timeout 300 python tools/sl_time.py C4 0 0 > gpurun_out/fx/c4_m$m.log 2>&1; echo "m=$m"; head -1 gpurun_out/fx/c4_m$m.log
  INSTA_FWDX=$m timeout 300 python tools/sl_time.py C4 1 0 > gpurun_out/fx/c4_lse_m$m.log 2>&1; head -1 gpurun_out/fx/c4_lse_m$m.log
done

mkdir -p gpurun_out/fx2
INSTA_FWDX=2 timeout 900 python -m pytest tests/test_gpu_parity.py -q -m gpu -x -k "not c4" > gpurun_out/fx2/par.log 2>&1; echo "parity rc=$?"; tail -1 gpurun_out/fx2/par.log
for m in 1 2; do
  INSTA_FWDX=$m timeout 300 python tools/sl_time.py C4 0 0 2>&1 | head -1
  INSTA_FWDX=$m timeout 300 python tools/sl_time.py C4 1 0 2>&1 | head -1
done
for v in nopf t512; do
  cd build_variants/$v
  for m in 1 2; do echo "$v m=$m"; INSTA_FWDX=$m timeout 300 python tools/sl_time.py C4 0 0 2>&1 | head -1; done
  cd ../..
done

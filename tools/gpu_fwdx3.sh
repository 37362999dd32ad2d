INSTA_FWDX=2 timeout 900 python -m pytest tests/test_gpu_parity.py -q -m gpu -x -k "not c4" 2>&1 | tail -1
for v in . build_variants/t512; do
  (cd $v; echo "$v"; for t in 0 1; do INSTA_FWDX=2 timeout 300 python tools/sl_time.py C4 $t 0 2>&1 | head -1; done)
done

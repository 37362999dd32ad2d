for v in t384 t512 t512g t640 t768g; do
  (cd build_variants/$v; echo "$v"; for rep in 1 2; do for t in 0 1; do INSTA_FWDX=2 timeout 300 python tools/sl_time.py C4 $t 0 2>&1 | head -1; done; done)
done

for v in orig e2 e3t640 e3t512 orig e3t640; do
  (cd build_variants/$v; echo "$v"; for t in 0 1; do timeout 300 python tools/sl_time.py C4 $t 0 2>&1 | head -1; done)
done

for v in . build_variants/cl5 build_variants/cl6 build_variants/cl8; do (cd $v; echo $v; timeout 300 python tools/clark_bench.py C4 2>&1 | tail -1); done

# forward schedules at C4 / C3: dataflow (0) vs level-synchronous sweep (3), per-level phase traces
mkdir -p gpurun_out/fp /tmp/tr0 /tmp/tr3
timeout 300 python tools/sl_time.py C4 0 0 > gpurun_out/fp/c4_s0.log 2>&1; echo "s0 rc=$?"
timeout 300 python tools/sl_time.py C4 0 3 > gpurun_out/fp/c4_s3.log 2>&1; echo "s3 rc=$?"
cd build_variants/phases
INSTA_SL_TRACE=/tmp/tr3 timeout 300 python tools/sl_time.py C4 0 3 > ../../gpurun_out/fp/c4_s3_phases.log 2>&1; echo "ph rc=$?"
INSTA_SL_TRACE=/tmp/tr3 timeout 300 python tools/sl_time.py C3 0 3 > ../../gpurun_out/fp/c3_s3_phases.log 2>&1; echo "ph3 rc=$?"
cd ../..
timeout 300 python tools/items_stats.py C4 > gpurun_out/fp/items_c4.log 2>&1

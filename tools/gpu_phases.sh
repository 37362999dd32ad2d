mkdir -p gpurun_out/ph
cd build_variants/phases
INSTA_SL_TRACE=../../gpurun_out/ph timeout 300 python tools/sl_time.py C4 0 3 > ../../gpurun_out/ph/c4.log 2>&1; echo "rc=$?"
cd ../..
python tools/phases.py gpurun_out/ph/sl_fwd.bin > gpurun_out/ph/fwd_phases.txt; head -40 gpurun_out/ph/fwd_phases.txt
rm -f gpurun_out/ph/*.bin.unused

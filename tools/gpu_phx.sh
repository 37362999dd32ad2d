mkdir -p gpurun_out/phx2
cd build_variants/phx
INSTA_FWDX=2 INSTA_SL_TRACE=../../gpurun_out/phx2 timeout 300 python tools/sl_time.py C4 0 0 > ../../gpurun_out/phx2/c4.log 2>&1; echo "rc=$?"
cd ../..
python tools/phases.py gpurun_out/phx2/sl_fwd.bin > gpurun_out/phx2/fwd_phases.txt; head -20 gpurun_out/phx2/fwd_phases.txt; sed -n 40,50p gpurun_out/phx2/fwd_phases.txt; sed -n 70,84p gpurun_out/phx2/fwd_phases.txt

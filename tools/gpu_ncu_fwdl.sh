mkdir -p gpurun_out/nf
timeout 900 ncu --set full --import-source on --clock-control none -k regex:"fwdl_kernel" -s 3 -c 1 -o gpurun_out/nf/fwdl python tools/sl_time.py C4 0 3 > gpurun_out/nf/ncu.log 2>&1; echo "ncu rc=$?"
tail -3 gpurun_out/nf/ncu.log

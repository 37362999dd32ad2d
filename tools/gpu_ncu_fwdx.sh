mkdir -p gpurun_out/nx
timeout 900 ncu --set full --import-source on --clock-control none -k regex:"fwdx_kernel" -s 3 -c 1 -o gpurun_out/nx/fwdx python tools/sl_time.py C4 0 3 > gpurun_out/nx/ncu.log 2>&1; echo "ncu rc=$?"
INSTA_FWDX=2 timeout 900 ncu --set full --import-source on --clock-control none -k regex:"fwdx_kernel" -s 3 -c 1 -o gpurun_out/nx/fwdx_flow python tools/sl_time.py C4 0 0 > gpurun_out/nx/ncu2.log 2>&1; echo "ncu rc=$?"

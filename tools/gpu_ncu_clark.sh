mkdir -p gpurun_out/cl
timeout 900 ncu --set full --import-source on --clock-control none -k regex:"cl_bwd_kernel" -s 200 -c 1 -o gpurun_out/cl/clbwd python tools/clark_bench.py C4 > gpurun_out/cl/ncu.log 2>&1; echo "ncu rc=$?"

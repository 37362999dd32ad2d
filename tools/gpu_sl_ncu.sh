# ncu --set full of one sweep forward and one sweep backward launch at C4 (hard mode)
timeout 900 ncu --set full --import-source on -k regex:"fwdl_kernel|bwdl_kernel" -s 8 -c 2 -o gpurun_out/sl_c4 python tools/sl_time.py C4 0 > gpurun_out/ncu_c4.log 2>&1; tail -3 gpurun_out/ncu_c4.log

# ncu full capture of one batched forward and one batched backward launch (C4, 32 scenarios)
timeout 900 ncu --set full --import-source on --clock-control none -k regex:"fwdb_kernel|bwdb_kernel" -s 2 -c 2 -o gpurun_out/prof_batch -f python tools/batch_debug.py C4 > gpurun_out/ncu_batch.log 2>&1; echo ncu=$?
tail -2 gpurun_out/ncu_batch.log

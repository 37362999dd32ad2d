timeout 600 ncu --set full --import-source on --clock-control none -k regex:"fwd_kernel" -s 2 -c 1 -o gpurun_out/prof_lse_fwd -f python bench.py --steps 1 --warmup 3 --tau 1 --e2e-steps 0 --no-cpu-baseline --batch-scenarios 0 --topk 0 --clark 0 > gpurun_out/ncu_lse.log 2>&1; echo ncu=$?
tail -2 gpurun_out/ncu_lse.log

# Profile evidence for profiles/ (run under gpurun): launch list of the bench
# command and one ncu --set full capture of the persistent kernels.
mkdir -p gpurun_out
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches.csv python bench.py --steps 2 --warmup 3 --e2e-steps 0 --no-cpu-baseline --batch-scenarios 64 > gpurun_out/ncu_list.log 2>&1; echo ncu1_rc=$?
timeout 900 ncu --set full --clock-control none --import-source on -k regex:"${KERN:-fwd_kernel|bwdf_kernel}" -s 2 -c 2 -o gpurun_out/prof_full -f python bench.py --steps 1 --warmup 3 --e2e-steps 0 --no-cpu-baseline --batch-scenarios 0 > gpurun_out/ncu_full.log 2>&1; echo ncu2_rc=$?
tail -2 gpurun_out/ncu_full.log

# quick GPU check of the sweep schedule: parity subset + C4 timings (schedules 0 and 2, hard and LSE)
set -x
timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_incremental.py -x -q -m "gpu and not slow" 2>&1 | tail -30 > gpurun_out/t1.log
cat gpurun_out/t1.log
for s in 0 2; do for tau in 0 1; do
timeout 300 python bench.py --steps 10 --warmup 3 --schedule $s --tau $tau --e2e-steps 0 --no-cpu-baseline --batch-scenarios 0 --topk 0 --clark 0 --incremental $((s==0)) > gpurun_out/b${s}_$tau.json 2> gpurun_out/b${s}_$tau.err
python -c "
import json,sys; d=json.loads(open('gpurun_out/b${s}_$tau.json').read().strip().split('\n')[-1]); print('sched $s tau $tau', d['fwd_ms'], d['bwd_ms'], d['fwd_bwd_ms'], d.get('incremental'))" || tail -5 gpurun_out/b${s}_$tau.err
done; done

mkdir -p gpurun_out
for T in 512 768 1024; do
  INSTA_NVCC_EXTRA="-DINSTA_FWD_THREADS=$T" python -c "from paper_conf_dac_lugklr25_b200 import build; build.build(force=True)" > /dev/null 2>&1
  echo "== T=$T"
  timeout 300 python -m pytest tests -m gpu -q -x -k "schedules or fold or tiny or dyadic or incremental" 2>&1 | tail -1
  for tau in 0 1; do timeout 300 python bench.py --steps 20 --warmup 5 --batch-scenarios 0 --no-cpu-baseline --e2e-steps 0 --tau $tau 2>/dev/null | python -c "
import json,sys; d=json.load(sys.stdin); print('tau', d['config']['tau'], 'fwd_ms', round(d['fwd_ms'],4), 'bwd_ms', round(d['bwd_ms'],4))"; done
done

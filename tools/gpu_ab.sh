# A/B of compile-time variants (run under gpurun): tools/gpu_ab.sh "NAME=FLAGS" ...
# Builds each variant as a full copy of the repo under build_variants/NAME,
# runs the GPU parity tests of the default build and times fwd/bwd at C4 for all.
set -x
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || tail -20 gpurun_out/build.log
for spec in "$@"; do
  n=${spec%%=*}; f=${spec#*=}
  d=build_variants/$n; rm -rf $d; mkdir -p $d
  cp -r paper_conf_dac_lugklr25_b200 include oracle bench.py $d/
  rm -f $d/paper_conf_dac_lugklr25_b200/libinsta.so
  (cd $d && INSTA_NVCC_EXTRA="$f" python -m paper_conf_dac_lugklr25_b200.build > /dev/null 2>&1); ls -la $d/paper_conf_dac_lugklr25_b200/libinsta.so
done
timeout 900 python -m pytest tests -m gpu -q -x ${TESTS:-tests/test_gpu_parity.py tests/test_gpu_incremental.py} > gpurun_out/ab_tests.log 2>&1; echo tests_rc=$?
tail -5 gpurun_out/ab_tests.log
A="--steps 20 --warmup 5 --batch-scenarios 0 --topk 0 --clark 0 --e2e-steps 0 --no-cpu-baseline ${BENCH_EXTRA:-}"
for rep in 1 2; do
  echo default; timeout 400 python bench.py $A | python -c "import json,sys; d=json.loads(sys.stdin.read()); print(d['fwd_ms'], d['bwd_ms'], d['roofline']['frac'])"
  for spec in "$@"; do n=${spec%%=*}; echo $n
    (cd build_variants/$n && timeout 400 python bench.py $A | python -c "import json,sys; d=json.loads(sys.stdin.read()); print(d['fwd_ms'], d['bwd_ms'], d['roofline']['frac'])"); done
done

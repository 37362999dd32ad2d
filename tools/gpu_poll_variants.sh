# re-poll back-off variants: fwd/bwd ms at C4 (hard)
A="--steps 20 --warmup 5 --batch-scenarios 0 --topk 0 --clark 0 --e2e-steps 0 --no-cpu-baseline"
echo default; timeout 400 python bench.py $A | python -c "import json,sys; d=json.loads(sys.stdin.read()); print(d['fwd_ms'], d['bwd_ms'])"
for v in p0 p5 p100; do echo $v; (cd build_variants/$v && timeout 400 python bench.py $A | python -c "import json,sys; d=json.loads(sys.stdin.read()); print(d['fwd_ms'], d['bwd_ms'])"); done

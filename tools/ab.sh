# A/B of library variants: ab_libs/<name>.so, alternated; parity tests on the first variant given in $TEST
# usage: VARIANTS="base wkill" TEST=wkill bash tools/ab.sh
mkdir -p gpurun_out
L=paper_conf_sc_gundaboluvt21_b200/libfastz.so
if [ -n "$TEST" ]; then
  cp ab_libs/$TEST.so $L
  timeout 900 python -m pytest tests -m gpu -x -q > gpurun_out/pytest_ab_$TEST.log 2>&1; tail -2 gpurun_out/pytest_ab_$TEST.log
fi
for rep in 1 2; do
  for v in $VARIANTS; do
    cp ab_libs/$v.so $L
    timeout 600 python bench.py --steps 3 --warmup 3 --no-cpu-baseline 2>/dev/null | tail -1 > gpurun_out/ab_$v.json
    python -c "import json; d=json.loads(open('gpurun_out/ab_$v.json').read()); print('$v', round(d['value'],1), 'inspect', round(d['stages_ms']['ms_inspect'],1), 'clk', d['clocks']['sm_mhz'])"
  done
done

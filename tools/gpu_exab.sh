L=paper_conf_sc_gundaboluvt21_b200/libfastz.so
cp $L /tmp/cur.so
TEST=ex6 VARIANTS="" bash tools/ab.sh
for v in cur ex6 ex7; do
  cp ab_libs/$v.so $L
  for c in 1 5; do echo -n "$v C$c "; timeout 900 python tools/config_run.py $c 4 2>/dev/null | tail -1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); print(d['stages_ms']['ms_execute'], d['stages_ms']['ms_total'], d['parity'])"; done
  timeout 600 python bench.py --steps 3 --warmup 3 --no-cpu-baseline 2>/dev/null | tail -1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('$v C2', d['stages_ms']['ms_execute'], d['ms_per_step'])"
done
cp /tmp/cur.so $L

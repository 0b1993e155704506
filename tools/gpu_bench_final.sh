mkdir -p gpurun_out
python -m paper_conf_sc_gundaboluvt21_b200.build > /dev/null
timeout 1200 python -m pytest tests -m gpu -x -q > gpurun_out/pytest_g.log 2>&1; tail -3 gpurun_out/pytest_g.log
for i in 1 2; do timeout 900 python bench.py > gpurun_out/bench_g$i.json 2> gpurun_out/bench_g$i.err; tail -2 gpurun_out/bench_g$i.err; python -c "import json; d=json.loads(open('gpurun_out/bench_g$i.json').read().strip().splitlines()[-1]); print(round(d['value'],1), round(d['e2e']['value'],1), round(d['roofline']['frac'],3), {k: round(v,2) for k,v in d['stages_ms'].items()}, d['genome_pair_wall_s'])"; done

mkdir -p gpurun_out
python -m paper_conf_sc_gundaboluvt21_b200.build > /dev/null
timeout 1500 python -m pytest tests -m gpu -x -q > gpurun_out/pytest_n.log 2>&1; tail -3 gpurun_out/pytest_n.log
timeout 600 python bench.py --steps 5 --warmup 3 --no-cpu-baseline > gpurun_out/bench_n.json 2> gpurun_out/bench_n.err
python -c "import json; d=json.loads(open('gpurun_out/bench_n.json').read().strip().splitlines()[-1]); print(round(d['value'],1), round(d['e2e']['value'],1), {k: round(v,2) for k,v in d['stages_ms'].items()}, d['gpu_launches'])"
bash tools/sanitize.sh

mkdir -p gpurun_out
python -m paper_conf_sc_gundaboluvt21_b200.build > /dev/null
timeout 1200 python -m pytest tests -m gpu -x -q > gpurun_out/pytest_tb2.log 2>&1; tail -2 gpurun_out/pytest_tb2.log
timeout 600 python bench.py --steps 5 --warmup 3 --no-cpu-baseline > gpurun_out/bench_tb2.json 2> gpurun_out/bench_tb2.err
python -c "import json; d=json.loads(open('gpurun_out/bench_tb2.json').read().strip().splitlines()[-1]); print(round(d['value'],1), round(d['e2e']['value'],1), {k: round(v,2) for k,v in d['stages_ms'].items()})"
timeout 900 python tools/config_run.py 1 16 2>&1 | tail -1
timeout 600 python tools/n_bench.py 2>&1 | tail -1

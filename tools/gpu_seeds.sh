# seeding tests + full GPU suite on the current build + seeding throughput
mkdir -p gpurun_out
python -m paper_conf_sc_gundaboluvt21_b200.build > /dev/null
timeout 900 python -m pytest tests/test_gpu_seeds.py -x -q > gpurun_out/pytest_seeds.log 2>&1; tail -3 gpurun_out/pytest_seeds.log
timeout 1200 python -m pytest tests -m gpu -q > gpurun_out/pytest_gpu_all.log 2>&1; tail -3 gpurun_out/pytest_gpu_all.log
timeout 900 python tools/seed_bench.py 2 300000 > gpurun_out/seed_bench.json 2> gpurun_out/seed_bench.err; cat gpurun_out/seed_bench.json; tail -3 gpurun_out/seed_bench.err
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/seed_launches.csv python tools/seed_bench.py 2 20000 > /dev/null 2>&1

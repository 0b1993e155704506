# one GPU session for the current HEAD: GPU tests, bench line, launch list, ncu full captures (inspector, executor)
# usage: TAG=r1c bash tools/gpu_round.sh
TAG=${TAG:-cur}
mkdir -p gpurun_out
python -m paper_conf_sc_gundaboluvt21_b200.build > /dev/null
timeout 1200 python -m pytest tests -m gpu -x -q > gpurun_out/pytest_gpu_$TAG.log 2>&1; tail -3 gpurun_out/pytest_gpu_$TAG.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke_$TAG.log 2>&1; tail -2 gpurun_out/smoke_$TAG.log
timeout 900 python bench.py > gpurun_out/bench_$TAG.json 2> gpurun_out/bench_$TAG.err; cat gpurun_out/bench_$TAG.json
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file gpurun_out/launches_$TAG.csv python bench.py --profile --no-cpu-baseline > /dev/null 2>&1
timeout 1500 ncu --set full --clock-control none --import-source on -k regex:k_inspect -s 1 -c 1 -o gpurun_out/insp_$TAG python bench.py --profile --no-cpu-baseline > gpurun_out/ncu_insp_$TAG.log 2>&1
timeout 1200 ncu --set full --clock-control none --import-source on -k regex:k_execute -s 1 -c 1 -o gpurun_out/exec_$TAG python bench.py --profile --no-cpu-baseline > gpurun_out/ncu_exec_$TAG.log 2>&1
ls gpurun_out

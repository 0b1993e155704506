# one GPU session: bench line, launch list, ncu full capture of the inspector
set -x
mkdir -p gpurun_out
python -m paper_conf_sc_gundaboluvt21_b200.build
timeout 900 python bench.py --steps 5 --warmup 3 > gpurun_out/bench.json 2> gpurun_out/bench.err; tail -5 gpurun_out/bench.err
cat gpurun_out/bench.json
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -c 60 --csv --log-file gpurun_out/launches.csv python bench.py --profile --no-cpu-baseline > gpurun_out/prof_bench.json 2>&1
timeout 1200 ncu --set full --clock-control none --import-source on -k regex:k_inspect -c 1 -o gpurun_out/insp python bench.py --profile --no-cpu-baseline > gpurun_out/ncu_full.log 2>&1
tail -3 gpurun_out/ncu_full.log
ls -la gpurun_out

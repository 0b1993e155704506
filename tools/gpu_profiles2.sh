mkdir -p gpurun_out
python -m paper_conf_sc_gundaboluvt21_b200.build > /dev/null
timeout 900 python bench.py > gpurun_out/bench_final.json 2> gpurun_out/bench_final.err
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file gpurun_out/launches_r1b.csv python bench.py --profile --no-cpu-baseline > /dev/null 2>&1
timeout 1500 ncu --set full --clock-control none --import-source on -k regex:k_inspect -s 1 -c 1 -o gpurun_out/insp_r1b python bench.py --profile --no-cpu-baseline > gpurun_out/ncu_r1b.log 2>&1
timeout 1200 ncu --set full --clock-control none --import-source on -k regex:k_execute -s 1 -c 1 -o gpurun_out/exec_r1b python bench.py --profile --no-cpu-baseline > gpurun_out/ncu_exec_r1b.log 2>&1
for c in 1 3 5 6; do timeout 1500 python tools/config_run.py $c 16 2>&1 | tail -1 >> gpurun_out/configs_r1b.jsonl; done
ls gpurun_out

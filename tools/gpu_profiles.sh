# Full-size profiles for profiles/: launch list (gpu__time_duration) of one bench step and one ncu --set full
# capture of the inspector at the bench configuration.
mkdir -p gpurun_out
python -m paper_conf_sc_gundaboluvt21_b200.build > /dev/null
FASTZ_INTPEAK_VERBOSE=1 python -c "
import paper_conf_sc_gundaboluvt21_b200 as f; print(f.fastz_int_peak(0, 300.0))" 2>&1 | tee gpurun_out/intpeak.txt
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file gpurun_out/launches_full.csv python bench.py --profile --no-cpu-baseline > gpurun_out/prof_bench_full.json 2>&1
timeout 1500 ncu --set full --clock-control none --import-source on -k regex:k_inspect -s 1 -c 1 -o gpurun_out/insp_full python bench.py --profile --no-cpu-baseline > gpurun_out/ncu_full.log 2>&1
tail -2 gpurun_out/ncu_full.log
timeout 1200 ncu --set full --clock-control none --import-source on -k regex:k_execute -c 1 -o gpurun_out/exec_full python bench.py --profile --no-cpu-baseline > gpurun_out/ncu_exec.log 2>&1
tail -2 gpurun_out/ncu_exec.log

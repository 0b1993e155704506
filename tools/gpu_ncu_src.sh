# one ncu --set full capture of the inspector (source-level SASS counters) on the C2 bench step
mkdir -p gpurun_out
python -m paper_conf_sc_gundaboluvt21_b200.build > /dev/null
timeout 1200 ncu --set full --clock-control none --import-source on -k regex:${KREGEX:-k_inspect} -c 1 -o gpurun_out/${TAG:-insp_src} python bench.py --profile --no-cpu-baseline > gpurun_out/${TAG:-insp_src}.log 2>&1
tail -3 gpurun_out/${TAG:-insp_src}.log

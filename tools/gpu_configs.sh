mkdir -p gpurun_out
python -m paper_conf_sc_gundaboluvt21_b200.build > /dev/null
timeout 1500 python -m pytest tests/test_gpu_fullsize.py -x -q > gpurun_out/pytest_full.log 2>&1; tail -3 gpurun_out/pytest_full.log
for c in ${CFGS:-1 5 3}; do timeout 1500 python tools/config_run.py $c ${NS:-16} 2>&1 | tail -2 | tee -a gpurun_out/configs.jsonl; done

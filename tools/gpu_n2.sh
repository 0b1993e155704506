mkdir -p gpurun_out
python -m paper_conf_sc_gundaboluvt21_b200.build > /dev/null
timeout 600 python -m pytest tests/test_gpu_parity.py tests/test_gpu_seeds.py -x -q -k "n_bases" > gpurun_out/pytest_n2.log 2>&1; tail -3 gpurun_out/pytest_n2.log
timeout 1500 python -m pytest tests -m gpu -q > gpurun_out/pytest_all_n.log 2>&1; tail -3 gpurun_out/pytest_all_n.log
bash tools/sanitize.sh

mkdir -p gpurun_out
python -m paper_conf_sc_gundaboluvt21_b200.build > /dev/null
timeout 600 python -m pytest tests/test_gpu_seeds.py -x -q > gpurun_out/pytest_seeds.log 2>&1; tail -3 gpurun_out/pytest_seeds.log
timeout 1200 python -m pytest tests -m gpu -x -q > gpurun_out/pytest_gpu_all.log 2>&1; tail -3 gpurun_out/pytest_gpu_all.log
cp paper_conf_sc_gundaboluvt21_b200/libfastz.so /tmp/cur.so
VARIANTS="t8u8 prof_m1 prof_m5 prof_m6" bash tools/ab.sh
cp /tmp/cur.so paper_conf_sc_gundaboluvt21_b200/libfastz.so

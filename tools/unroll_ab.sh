# A/B of the steady-state unroll factor (rebuilds the library with -DSTEADY_UNROLL=8 into a temp copy)
set -e
python -m paper_conf_sc_gundaboluvt21_b200.build > /dev/null
cp paper_conf_sc_gundaboluvt21_b200/libfastz.so /tmp/lib4.so
cd paper_conf_sc_gundaboluvt21_b200/csrc && /usr/local/cuda/bin/nvcc -gencode arch=compute_100a,code=sm_100a -lineinfo -O3 -std=c++17 -Xcompiler -fPIC -shared -diag-suppress 177 -DSTEADY_UNROLL=8 -o /tmp/lib8.so api.cu kernels.cu intpeak.cu && cd ../..
for v in 4 8 4 8; do cp /tmp/lib$v.so paper_conf_sc_gundaboluvt21_b200/libfastz.so; FASTZ_R=4 timeout 600 python bench.py --steps 3 --warmup 2 --no-cpu-baseline 2>/dev/null | python -c "import json,sys; d=json.loads(sys.stdin.read().splitlines()[-1]); print('unroll $v', round(d['value'],1), 'inspect', round(d['stages_ms']['ms_inspect'],1))"; done
cp /tmp/lib4.so paper_conf_sc_gundaboluvt21_b200/libfastz.so
for bb in 3 7; do FASTZ_BLOCK_BIN=$bb timeout 900 python tools/config_run.py 1 4 2>&1 | tail -1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('C1 block_bin $bb', d['stages_ms'], d['parity'])"; done

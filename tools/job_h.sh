python tools/config_sweep.py 1 2 3 5 6 > gpurun_out/h_sweep.jsonl 2> gpurun_out/h_sweep.err
FASTZ_LIB=ab_libs/libfastz_e5.so python tools/config_sweep.py 1 2 3 5 > gpurun_out/h_sweep_e5.jsonl 2> gpurun_out/h_sweep_e5.err
for esc in 16 64; do FASTZ_ESCALATE_STRIPS=$esc python tools/config_sweep.py 1 > gpurun_out/h_esc_$esc.jsonl 2>&1; done
cat gpurun_out/h_sweep.jsonl gpurun_out/h_sweep_e5.jsonl gpurun_out/h_esc_*.jsonl

python tools/config_sweep.py 2 3 5 1 6 > gpurun_out/n_sweep.jsonl 2> gpurun_out/n_sweep.err
FASTZ_INSPECT_ORDER=0 python tools/config_sweep.py 2 > gpurun_out/n_sweep_noorder.jsonl 2>&1
cat gpurun_out/n_sweep.jsonl gpurun_out/n_sweep_noorder.jsonl

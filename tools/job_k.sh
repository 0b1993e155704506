# inspector order A/B: predicted-longest-first (default) vs seed order; plus the class-label upper bound on C3
python tools/config_sweep.py 1 2 3 5 6 > gpurun_out/k_sweep_order.jsonl 2> gpurun_out/k_sweep_order.err
FASTZ_INSPECT_ORDER=0 python tools/config_sweep.py 1 2 3 5 6 > gpurun_out/k_sweep_noorder.jsonl 2> gpurun_out/k_sweep_noorder.err
FASTZ_INSPECT_ORDER=0 python tools/order_probe.py 3 > gpurun_out/k_order_probe_c3.txt 2>&1
cat gpurun_out/k_sweep_order.jsonl gpurun_out/k_sweep_noorder.jsonl gpurun_out/k_order_probe_c3.txt
MODE=tests TAG=k bash tools/gpu.sh

python tools/config_sweep.py 1 2 3 5 6 > gpurun_out/i_sweep.jsonl 2> gpurun_out/i_sweep.err
FASTZ_LIB=$PWD/ab_libs/libfastz_e5.so python tools/config_sweep.py 1 2 3 5 > gpurun_out/i_sweep_e5.jsonl 2> gpurun_out/i_sweep_e5.err
cat gpurun_out/i_sweep.jsonl gpurun_out/i_sweep_e5.jsonl
MODE=tests TAG=i bash tools/gpu.sh

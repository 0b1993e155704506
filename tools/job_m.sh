python tools/config_sweep.py 3 2 5 1 > gpurun_out/m_sweep.jsonl 2> gpurun_out/m_sweep.err
cat gpurun_out/m_sweep.jsonl
MODE=tests TAG=m bash tools/gpu.sh

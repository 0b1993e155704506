MODE=tests TAG=j bash tools/gpu.sh
MODE=bench TAG=j bash tools/gpu.sh
MODE=launch TAG=j BENCH_ARGS="--no-secondary --no-genome-pair" bash tools/gpu.sh
MODE=ncu TAG=j_insp KREGEX=k_inspect BENCH_ARGS="--no-secondary --no-genome-pair" bash tools/gpu.sh

bash tools/sanitize.sh
MODE=tests TAG=l PYTEST_ARGS="tests/test_gpu_parity.py tests/test_gpu_wide.py tests/test_gpu_abi.py" bash tools/gpu.sh

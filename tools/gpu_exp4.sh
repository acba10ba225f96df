mkdir -p gpurun_out
./tools/mufu_bench
DJINN_LRN_POOL=1 timeout 600 python -m pytest tests/test_parity_gpu.py tests/test_fullsize_gpu.py -m gpu -q -k "imc" --timeout 300 2>&1 | grep -E "passed|failed|Error|assert" | head

mkdir -p gpurun_out
DJINN_LRN_POOL=1 timeout 600 python -m pytest tests/test_parity_gpu.py tests/test_fullsize_gpu.py -m gpu -q -k "imc" --timeout 300 2>&1 | tail -2
DJINN_LRN_POOL=1 TAG=lrnpool timeout 300 python tools/op_times.py imc bf16 2>&1 | grep -E "conv|norm|pool|total"
DJINN_LRN_POOL=1 TAG=lrnpool timeout 300 python tools/op_times.py imc fp16 2>&1 | grep -E "norm|total"
timeout 300 python tools/op_times.py imc bf16 2>&1 | grep -E "conv1|conv2|pool1|pool2|total"

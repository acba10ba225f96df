mkdir -p gpurun_out
timeout 900 python -m pytest tests -m gpu -q -x --timeout 600 2>&1 | tail -2
DJINN_LRN_POOL=3 timeout 600 python -m pytest tests/test_parity_gpu.py tests/test_fullsize_gpu.py -m gpu -q -k "imc" --timeout 300 2>&1 | tail -1
for m in 0 3; do DJINN_LRN_POOL=$m TAG=mask$m timeout 300 python tools/op_times.py imc bf16 2>&1 | grep -E "conv1|conv2|norm|pool1|pool2|total"; done

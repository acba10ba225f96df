mkdir -p gpurun_out
DJINN_LRN_POOL=1 TAG=lrnpool timeout 300 python tools/op_times.py imc bf16 2>&1 | tail -16
DJINN_LRN_POOL=1 TAG=lrnpool timeout 300 python tools/op_times.py imc fp16 2>&1 | grep -E "conv1|conv2|norm|pool"

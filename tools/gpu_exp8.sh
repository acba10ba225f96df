mkdir -p gpurun_out
timeout 900 python -m pytest tests -m gpu -q -x --timeout 600 2>&1 | tail -2
timeout 300 python tools/op_times.py imc bf16 2>&1 | grep -E "conv|norm|pool1|pool2|fc|total"
DJINN_LRN_POOL=1 TAG=lrnpool timeout 300 python tools/op_times.py imc bf16 2>&1 | grep -E "conv1|conv2|norm|total"
for a in face asr dig pos; do timeout 300 python tools/op_times.py $a bf16 2>&1 | grep -E "gemm|total"; done

mkdir -p gpurun_out
timeout 900 python -m pytest tests -m gpu -q -x --timeout 600 2>&1 | tail -2
for m in 0 2; do DJINN_LRN_POOL=$m TAG=mask$m timeout 300 python tools/op_times.py imc bf16 2>&1 | grep -E "conv1|conv2|norm|pool|total"; done
for a in face dig; do timeout 300 python tools/op_times.py $a bf16 2>&1 | grep -E "pool|M2|total"; done

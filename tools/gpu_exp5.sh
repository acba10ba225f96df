mkdir -p gpurun_out
timeout 900 python -m pytest tests -m gpu -q -x --timeout 600 2>&1 | tail -2
for ts in 2 0; do
  DJINN_TSLOTS=$ts TAG=tslots$ts timeout 300 python tools/op_times.py imc bf16 2>&1 | grep -E "conv|norm|pool1|pool2|total"
  DJINN_TSLOTS=$ts DJINN_LRN_POOL=1 TAG=lrnpool-tslots$ts timeout 300 python tools/op_times.py imc bf16 2>&1 | grep -E "conv1|conv2|norm|total"
  DJINN_TSLOTS=$ts TAG=tslots$ts timeout 300 python tools/op_times.py face bf16 2>&1 | grep -E "C1|C3|L4|L5|L6|F7|total"
  DJINN_TSLOTS=$ts TAG=tslots$ts timeout 300 python tools/op_times.py dig bf16 2>&1 | grep -E "conv|ip|total"
done

mkdir -p gpurun_out
L=$PWD/paper_conf_isca_hauswaldklclmdm15_b200
DJINN_LRN_POOL=1 timeout 600 python -m pytest tests/test_parity_gpu.py tests/test_fullsize_gpu.py -m gpu -q -k "imc" --timeout 300 2>&1 | tail -4
DJINN_LRN_POOL=1 TAG=lrnpool timeout 300 python tools/op_times.py imc bf16 2>&1 | grep -E "conv|norm|pool|pack|total"
DJINN_LRN_POOL=1 DJINN_LIB=$L/libdjinn_nostore.so TAG=lrnpool-nostore timeout 300 python tools/op_times.py imc bf16 2>&1 | grep -E "conv1|conv2"
DJINN_LIB=$L/libdjinn_nostore.so TAG=nostore timeout 300 python tools/op_times.py imc bf16 2>&1 | grep -E "conv|total"
DJINN_LIB=$L/libdjinn_nostore.so TAG=nostore timeout 300 python tools/op_times.py face bf16 2>&1 | grep -E "C1|C3|L4|total"

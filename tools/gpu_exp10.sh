mkdir -p gpurun_out
L=$PWD/paper_conf_isca_hauswaldklclmdm15_b200
DJINN_LRN_POOL=1 DJINN_LIB=$L/libdjinn_poly.so TAG=poly timeout 300 python tools/op_times.py imc bf16 2>&1 | grep -E "norm"
DJINN_LRN_POOL=1 DJINN_LIB=$L/libdjinn_poly.so timeout 600 python -m pytest tests/test_fullsize_gpu.py -m gpu -q -k "imc" --timeout 300 2>&1 | tail -1
DJINN_LRN_POOL=1 timeout 600 /usr/local/cuda/bin/ncu --set full --clock-control none --import-source on -k regex:lrn_pool -s 0 -c 1 \
  -o gpurun_out/imc_lrnpool1b python tools/run_app.py imc bf16 1024 1 > gpurun_out/ncu_lp.log 2>&1

mkdir -p gpurun_out
L=$PWD/paper_conf_isca_hauswaldklclmdm15_b200
DJINN_LRN_POOL=1 DJINN_LIB=$L/libdjinn_stats.so timeout 300 python tools/op_times.py imc bf16 1024 1 2>&1 | grep "tc BN" | head -6
DJINN_LIB=$L/libdjinn_stats.so timeout 300 python tools/op_times.py face bf16 256 1 2>&1 | grep "tc BN" | head -3
DJINN_LRN_POOL=1 timeout 600 /usr/local/cuda/bin/ncu --set full --clock-control none --import-source on -k regex:tc_gemm -s 0 -c 1 \
  -o gpurun_out/imc_c1_plain python tools/run_app.py imc bf16 1024 1 > gpurun_out/ncu_c1p.log 2>&1
DJINN_LRN_POOL=1 timeout 600 /usr/local/cuda/bin/ncu --set full --clock-control none --import-source on -k regex:lrn_pool -s 0 -c 1 \
  -o gpurun_out/imc_lrnpool1 python tools/run_app.py imc bf16 1024 1 > gpurun_out/ncu_lp.log 2>&1
tail -1 gpurun_out/ncu_c1p.log gpurun_out/ncu_lp.log

# ncu full capture of IMC conv1 + conv2 (first two tc_gemm launches of one forward)
mkdir -p gpurun_out
timeout 600 /usr/local/cuda/bin/ncu --set full --clock-control none --import-source on -k regex:tc_gemm -s 0 -c 2 \
  -o gpurun_out/imc_slab python tools/run_app.py imc bf16 1024 1 > gpurun_out/ncu_imc.log 2>&1
tail -2 gpurun_out/ncu_imc.log

/usr/local/cuda/bin/ncu --set full --clock-control none --import-source on -k regex:tc_gemm -s 0 -c 1 -o gpurun_out/imc_c1 python tools/run_app.py imc bf16 1024 1 > gpurun_out/ncu_imc_c1.log 2>&1
timeout 600 python -m pytest tests/test_parity_gpu.py tests/test_fullsize_gpu.py -m gpu -q --timeout 200 2>&1 | tail -1

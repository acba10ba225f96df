NCU=/usr/local/cuda/bin/ncu
$NCU --set full --clock-control none --import-source on -k regex:tc_gemm -s 0 -c 3 -o gpurun_out/imc_tc3 python tools/run_app.py imc bf16 1024 1 > gpurun_out/ncu_imc3.log 2>&1
$NCU --set full --clock-control none --import-source on -k regex:tc_gemm -s 1 -c 1 -o gpurun_out/asr_tc3 python tools/run_app.py asr bf16 8192 1 > gpurun_out/ncu_asr3.log 2>&1
timeout 300 python -m pytest tests/test_parity_gpu.py -m gpu -q -x -k "fp32 and imc" 2>&1 | grep -E "Error|error" | head -5

set -x
NCU=/usr/local/cuda/bin/ncu
$NCU --set full --clock-control none --import-source on -k regex:tc_gemm -s 3 -c 4 -o gpurun_out/face_tc python tools/run_app.py face bf16 256 1 > gpurun_out/ncu_face.log 2>&1
$NCU --set full --clock-control none --import-source on -k regex:tc_gemm -s 0 -c 3 -o gpurun_out/imc_tc python tools/run_app.py imc bf16 1024 1 > gpurun_out/ncu_imc.log 2>&1
$NCU --set full --clock-control none --import-source on -k regex:tc_gemm -s 1 -c 2 -o gpurun_out/asr_tc python tools/run_app.py asr bf16 8192 1 > gpurun_out/ncu_asr.log 2>&1
ls -la gpurun_out

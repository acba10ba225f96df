NCU=/usr/local/cuda/bin/ncu
$NCU --set full --clock-control none --import-source on -k regex:tc_gemm -s 0 -c 2 -o gpurun_out/face_tc4 python tools/run_app.py face bf16 256 1 > gpurun_out/ncu_face4.log 2>&1

# Per-op times of every app, no-epilogue + role-timing variants of IMC/FACE, ncu full capture of IMC conv1
mkdir -p gpurun_out
L=$PWD/paper_conf_isca_hauswaldklclmdm15_b200
for a in imc face asr pos dig; do timeout 300 python tools/op_times.py $a bf16; done > gpurun_out/op_all.txt 2>&1
for a in imc face; do DJINN_LIB=$L/libdjinn_noepi.so TAG=noepi timeout 300 python tools/op_times.py $a bf16 2>&1 | grep gemm; done > gpurun_out/diag_noepi.txt
for a in imc:1024 face:256; do DJINN_LIB=$L/libdjinn_stats.so timeout 300 python tools/op_times.py ${a%%:*} bf16 ${a##*:} 1 2>&1 | grep "tc BN" | tail -30; done > gpurun_out/diag_stats.txt
timeout 600 /usr/local/cuda/bin/ncu --set full --clock-control none --import-source on -k regex:tc_gemm -s 0 -c 1 \
  -o gpurun_out/imc_c1 python tools/run_app.py imc bf16 1024 1 > gpurun_out/ncu_imc_c1.log 2>&1
tail -2 gpurun_out/ncu_imc_c1.log

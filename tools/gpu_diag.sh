# Diagnostic: role timing (stats build) and no-epilogue timing of IMC / FACE
mkdir -p gpurun_out
L=$PWD/paper_conf_isca_hauswaldklclmdm15_b200
for a in imc face; do DJINN_LIB=$L/libdjinn_noepi.so TAG=noepi timeout 300 python tools/op_times.py $a bf16 2>&1 | grep gemm; done > gpurun_out/diag_noepi.txt
for a in imc:1024 face:256; do DJINN_LIB=$L/libdjinn_stats.so timeout 300 python tools/op_times.py ${a%%:*} bf16 ${a##*:} 1 2>&1 | grep "tc BN" | tail -30; done > gpurun_out/diag_stats.txt

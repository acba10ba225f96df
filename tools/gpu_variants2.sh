# Per-op times of IMC / FACE under: default build, no-epilogue, stream-only (no MMA, no epilogue)
mkdir -p gpurun_out
L=$PWD/paper_conf_isca_hauswaldklclmdm15_b200
for v in libdjinn libdjinn_noepi libdjinn_stream; do
  for a in imc face; do DJINN_LIB=$L/$v.so TAG=$v timeout 300 python tools/op_times.py $a bf16 2>&1 | grep -E "gemm|total|pack|pool"; done
done > gpurun_out/variants2.txt
for a in imc:1024 face:256; do DJINN_LIB=$L/libdjinn_stats.so timeout 300 python tools/op_times.py ${a%%:*} bf16 ${a##*:} 1 2>&1 | grep "tc BN" | tail -30; done > gpurun_out/diag_stats.txt

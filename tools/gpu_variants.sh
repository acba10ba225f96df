# Diagnostic: per-op times of IMC / FACE under the diagnostic builds (no epilogue / no MMA / no
# stores) and the role-timing build (DJINN_TC_STATS).
mkdir -p gpurun_out
L=$PWD/paper_conf_isca_hauswaldklclmdm15_b200
for v in libdjinn libdjinn_noepi libdjinn_nomma libdjinn_nostore; do
  for a in imc face; do DJINN_LIB=$L/$v.so TAG=$v timeout 300 python tools/op_times.py $a bf16 2>&1 | grep -v "^\[.*\] *$" ; done
done > gpurun_out/variants.txt
DJINN_LIB=$L/libdjinn_stats.so timeout 300 python tools/op_times.py imc bf16 1024 1 > gpurun_out/stats_imc.txt 2>&1
DJINN_LIB=$L/libdjinn_stats.so timeout 300 python tools/op_times.py face bf16 256 1 > gpurun_out/stats_face.txt 2>&1

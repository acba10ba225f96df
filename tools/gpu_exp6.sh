mkdir -p gpurun_out
L=$PWD/paper_conf_isca_hauswaldklclmdm15_b200
for v in noepi nostore coal; do
  DJINN_LIB=$L/libdjinn_$v.so TAG=$v timeout 300 python tools/op_times.py imc bf16 2>&1 | grep -E "conv|fc6|fc7"
  DJINN_LRN_POOL=1 DJINN_LIB=$L/libdjinn_$v.so TAG=lrnpool-$v timeout 300 python tools/op_times.py imc bf16 2>&1 | grep -E "conv1|conv2"
  DJINN_LIB=$L/libdjinn_$v.so TAG=$v timeout 300 python tools/op_times.py face bf16 2>&1 | grep -E "C1|C3|L4|F7"
  DJINN_LIB=$L/libdjinn_$v.so TAG=$v timeout 300 python tools/op_times.py asr bf16 2>&1 | grep -E "a1|out"
done

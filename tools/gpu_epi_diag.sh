# Plain-epilogue diagnosis (IMC, DJINN_LRN_POOL=3 so conv1 has a bias+ReLU epilogue):
# full / no epilogue / no stores / TMEM loads only / coalesced-address stores (wrong results).
mkdir -p gpurun_out
L=$PWD/paper_conf_isca_hauswaldklclmdm15_b200
{
for v in libdjinn libdjinn_noepi libdjinn_nostore libdjinn_ldonly libdjinn_coal; do
  DJINN_LRN_POOL=3 DJINN_LIB=$L/$v.so TAG=$v timeout 300 python tools/op_times.py imc bf16 1024 10 2>&1 | grep -E "conv|total"
done
} > gpurun_out/epi_diag.txt 2>&1
cat gpurun_out/epi_diag.txt

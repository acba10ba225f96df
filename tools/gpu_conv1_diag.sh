# IMC conv1(+norm1) diagnosis: per-op times with diagnostic builds (no epilogue / no stores /
# LRN without MUFU / one MUFU / no B loads) and with the LRN placement masks.
mkdir -p gpurun_out
L=$PWD/paper_conf_isca_hauswaldklclmdm15_b200
{
for v in libdjinn libdjinn_noepi libdjinn_nostore libdjinn_lrn0 libdjinn_lrn1 libdjinn_nob; do
  DJINN_LIB=$L/$v.so TAG=$v timeout 300 python tools/op_times.py imc bf16 1024 10 2>&1 | grep -E "conv1|pool1|total"
done
for m in 0 3; do DJINN_LRN_POOL=$m TAG=mask$m timeout 300 python tools/op_times.py imc bf16 1024 10 2>&1 | grep -E "conv1|norm1|pool1|total"; done
} > gpurun_out/conv1_diag.txt 2>&1
cat gpurun_out/conv1_diag.txt

# Epilogue warpgroups: default (3 for LRN epilogues, 2 elsewhere; 3 loader warps), 2 everywhere
# (same build), and the 2-warpgroup build (4 loader warps).  Then GPU parity.
mkdir -p gpurun_out
L=$PWD/paper_conf_isca_hauswaldklclmdm15_b200
{
for cfg in "libdjinn:0" "libdjinn:2" "libdjinn:3" "libdjinn_epi2:0"; do
  v=${cfg%%:*}; w=${cfg##*:}
  for a in imc face asr dig pos; do DJINN_EPI_WG=$w DJINN_LIB=$L/$v.so TAG=$v/$w timeout 300 python tools/op_times.py $a bf16 2>&1 | grep -E "gemm|total"; done
done
} > gpurun_out/epiwg.txt 2>&1
timeout 900 python -m pytest tests -m gpu -q --timeout 600 > gpurun_out/pytest_gpu.log 2>&1; tail -3 gpurun_out/pytest_gpu.log

# Per-op conv times: stream-only (no MMA / epilogue), MMA-only (no B loads, no epilogue), no-epilogue
mkdir -p gpurun_out
L=$PWD/paper_conf_isca_hauswaldklclmdm15_b200
for v in libdjinn_mmaonly libdjinn_mmaepi; do
  for a in imc face; do DJINN_LIB=$L/$v.so TAG=$v timeout 300 python tools/op_times.py $a bf16 2>&1 | grep -E "conv|C1|C3"; done
done > gpurun_out/variants3.txt

# Parity + per-op conv times of the default build and the MMA-only diagnostic build
mkdir -p gpurun_out
[ -n "$NOTEST" ] || { timeout 900 python -m pytest tests -m gpu -q -x --timeout 600 > gpurun_out/pytest_gpu.log 2>&1; tail -2 gpurun_out/pytest_gpu.log; }
L=$PWD/paper_conf_isca_hauswaldklclmdm15_b200
for v in libdjinn libdjinn_mmaonly; do
  for a in imc face; do DJINN_LIB=$L/$v.so TAG=$v timeout 300 python tools/op_times.py $a bf16 2>&1 | grep -E "conv|C1|C3|total"; done
done

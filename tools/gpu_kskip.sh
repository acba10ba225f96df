# Zero-K-sub-step skipping in slab convs, same box: the build without the skip test, then the
# default build with DJINN_KSKIP=0 (off) and default; twice each (box noise).
mkdir -p gpurun_out
L=$PWD/paper_conf_isca_hauswaldklclmdm15_b200
{
for rep in 1 2; do
DJINN_LIB=$L/libdjinn_nokskip.so TAG=nocode timeout 300 python tools/op_times.py imc bf16 1024 10 2>&1 | grep -E "conv|total"
for k in 0 1; do DJINN_KSKIP=$k TAG=kskip$k timeout 300 python tools/op_times.py imc bf16 1024 10 2>&1 | grep -E "conv|total"; done
done
} > gpurun_out/kskip.txt 2>&1
nvidia-smi --query-gpu=clocks.sm,clocks.max.sm,power.draw,temperature.gpu --format=csv >> gpurun_out/kskip.txt
cat gpurun_out/kskip.txt

# Role timing (stats build, CTA 0) of IMC conv1: default (LRN epilogue) and plain epilogue (mask 3).
mkdir -p gpurun_out
L=$PWD/paper_conf_isca_hauswaldklclmdm15_b200
{
DJINN_LIB=$L/libdjinn_stats.so timeout 300 python tools/op_times.py imc bf16 1024 1 2>&1 | grep "tc BN" | head -6
echo mask3
DJINN_LRN_POOL=3 DJINN_LIB=$L/libdjinn_stats.so timeout 300 python tools/op_times.py imc bf16 1024 1 2>&1 | grep "tc BN" | head -6
} > gpurun_out/conv1_stats.txt 2>&1
cat gpurun_out/conv1_stats.txt

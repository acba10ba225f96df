# Zero-K-sub-step skipping (compile-time 3-MMA K blocks for 48-of-64-channel taps): IMC per-op
# times with DJINN_KSKIP=0 (off) / default, twice each, then IMC GPU parity.
mkdir -p gpurun_out
{
for rep in 1 2; do
for k in 0 1; do DJINN_KSKIP=$k TAG=kskip$k timeout 300 python tools/op_times.py imc bf16 1024 10 2>&1 | grep -E "conv|total"; done
done
} > gpurun_out/kskip.txt 2>&1
timeout 900 python -m pytest tests -m gpu -q --timeout 600 -k "imc or chunk" > gpurun_out/pytest_kskip.log 2>&1; tail -3 gpurun_out/pytest_kskip.log
cat gpurun_out/kskip.txt

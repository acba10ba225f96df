# IMC per-op times (twice) and the IMC GPU parity tests.
mkdir -p gpurun_out
{ for rep in 1 2; do timeout 300 python tools/op_times.py imc bf16 1024 10 2>&1 | grep -E "conv|pool|pack|total"; done; } > gpurun_out/imc_quick.txt 2>&1
timeout 900 python -m pytest tests -m gpu -q --timeout 600 -k "imc" > gpurun_out/pytest_imc.log 2>&1; tail -2 gpurun_out/pytest_imc.log
cat gpurun_out/imc_quick.txt

# IMC per-op times (default, then DJINN_PACK_ROWS=0) and the IMC / forward16 GPU parity tests.
mkdir -p gpurun_out
{ for v in 1 0; do DJINN_PACK_ROWS=$v TAG=packrows$v timeout 300 python tools/op_times.py imc bf16 1024 10 2>&1 | grep -E "conv1|pool1|pack|total"; done; } > gpurun_out/imc_quick.txt 2>&1
timeout 900 python -m pytest tests -m gpu -q --timeout 600 -k "imc or forward16 or pack" > gpurun_out/pytest_imc.log 2>&1; tail -2 gpurun_out/pytest_imc.log
cat gpurun_out/imc_quick.txt

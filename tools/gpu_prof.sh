# One GPU session: parity tests, per-op times, ncu full captures of IMC conv1 / conv2.
set -u
mkdir -p gpurun_out
timeout 900 python -m pytest tests -m gpu -q -rf --timeout 600 -x > gpurun_out/pytest_gpu.log 2>&1; tail -3 gpurun_out/pytest_gpu.log
for a in imc face dig; do timeout 300 python tools/op_times.py $a bf16 > gpurun_out/op_$a.txt 2>&1; done
tail -n 30 gpurun_out/op_*.txt
timeout 600 /usr/local/cuda/bin/ncu --set full --clock-control none --import-source on -k regex:tc_gemm -s 0 -c 2 \
  -o gpurun_out/imc_c12 python tools/run_app.py imc bf16 1024 1 > gpurun_out/ncu_imc.log 2>&1
tail -3 gpurun_out/ncu_imc.log

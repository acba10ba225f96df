# Quick GPU check: parity tests (-x) and per-op times of the conv-heavy apps.
mkdir -p gpurun_out
timeout 900 python -m pytest tests -m gpu -q -x --timeout 600 > gpurun_out/pytest_gpu.log 2>&1; tail -4 gpurun_out/pytest_gpu.log
for a in ${APPS:-imc face}; do timeout 300 python tools/op_times.py $a bf16 2>&1 | tail -16; done

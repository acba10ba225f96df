# One GPU session: tests, bench, ncu launch list of the bench command, full capture of the top kernel.
# usage: TOP_APP=imc TOP_SKIP=0 bash tools/gpu_round.sh   (TOP_SKIP = tc_gemm launches to skip in that app)
set -u
mkdir -p gpurun_out
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,power.draw --format=csv > gpurun_out/gpu.txt
timeout 900 python -m pytest tests -m gpu -q -rf --timeout 600 > gpurun_out/pytest_gpu.log 2>&1; tail -3 gpurun_out/pytest_gpu.log
timeout 900 python bench.py > gpurun_out/bench.json 2> gpurun_out/bench.err; tail -c 300 gpurun_out/bench.json
DJINN_BENCH_ALLOW_SHORT=1 timeout 900 /usr/local/cuda/bin/ncu --metrics gpu__time_duration.sum --clock-control none --csv \
  --log-file gpurun_out/launches.csv python bench.py --steps 2 --warmup 3 --no-cpu-baseline --no-e2e > gpurun_out/ncu_bench.log 2>&1
timeout 600 /usr/local/cuda/bin/ncu --set full --clock-control none --import-source on -k regex:${TOP_KERNEL:-tc_gemm} -s ${TOP_SKIP:-0} -c 1 \
  -o gpurun_out/top_kernel python tools/run_app.py ${TOP_APP:-imc} bf16 ${TOP_ROWS:-1024} 1 > gpurun_out/ncu_top.log 2>&1
ls -la gpurun_out | tail -12

# One GPU session: tests, bench, ncu launch list of the bench command, full captures of the
# first tc_gemm launches of an app (TOP_SKIPS = tc_gemm launches to skip, one report each).
# usage: TOP_APP=imc TOP_SKIPS="0 1" bash tools/gpu_round.sh
set -u
mkdir -p gpurun_out
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,power.draw --format=csv > gpurun_out/gpu.txt
timeout 900 python -m pytest tests -m gpu -q -rf --timeout 600 > gpurun_out/pytest_gpu.log 2>&1; tail -3 gpurun_out/pytest_gpu.log
timeout 900 python bench.py > gpurun_out/bench.json 2> gpurun_out/bench.err; tail -c 300 gpurun_out/bench.json
DJINN_BENCH_ALLOW_SHORT=1 timeout 900 /usr/local/cuda/bin/ncu --metrics gpu__time_duration.sum --clock-control none --csv \
  --log-file gpurun_out/launches.csv python bench.py --steps 2 --warmup 3 --no-cpu-baseline --no-e2e --no-concurrent --no-ids > gpurun_out/ncu_bench.log 2>&1
for sk in ${TOP_SKIPS:-0}; do
timeout 600 /usr/local/cuda/bin/ncu --set full --clock-control none --import-source on -k regex:${TOP_KERNEL:-tc_gemm} -s $sk -c 1 \
  -o gpurun_out/top_kernel_s$sk python tools/run_app.py ${TOP_APP:-imc} bf16 ${TOP_ROWS:-1024} 1 > gpurun_out/ncu_top_s$sk.log 2>&1
done
ls -la gpurun_out | tail -12

#!/bin/bash
# round-2 final evidence: bench line, ncu launch list + per-kernel ncu summaries, sanitizers
mkdir -p gpurun_out
timeout 900 python bench.py --steps 20 --warmup 5 --profile-json gpurun_out/bench_ops.json > gpurun_out/bench.json 2> gpurun_out/bench.err
echo "bench rc=$?" >> gpurun_out/bench.err
rm -f gpurun_out/ncu_kernels.jsonl
bash tools/gpu_profiles.sh

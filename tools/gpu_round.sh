#!/bin/bash
# Full GPU round: -m gpu tests, smoke, a default bench line (logs under gpurun_out/).
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke.log 2>&1; echo "smoke rc=$?" >> gpurun_out/smoke.log
DJINN_PARITY_LOG=gpurun_out/parity_full.jsonl timeout 2400 python -m pytest tests -m gpu -q -rfEx -p no:cacheprovider > gpurun_out/pytest_gpu.log 2>&1
echo "rc=$?" >> gpurun_out/pytest_gpu.log
timeout 900 python bench.py --steps 20 --warmup 5 --profile-json gpurun_out/bench_ops.json > gpurun_out/bench.json 2> gpurun_out/bench.err
echo "bench rc=$?" >> gpurun_out/bench.err

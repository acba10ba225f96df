#!/bin/bash
# Full-size parity (every bench-batch row vs the oracle) with per-(app,precision) stats logged.
mkdir -p gpurun_out
nproc > gpurun_out/nproc.txt
DJINN_PARITY_LOG=gpurun_out/parity_full.jsonl timeout 1500 python -m pytest tests/test_fullsize_gpu.py -q -s -p no:cacheprovider > gpurun_out/pytest_full.log 2>&1
echo "rc=$?" >> gpurun_out/pytest_full.log

#!/bin/bash
# Cluster dense+softmax kernel: parity tests, then ASR per-op times fused vs unfused.
mkdir -p gpurun_out
timeout 600 python -m pytest tests/test_fused_gpu.py -x -q -s -p no:cacheprovider > gpurun_out/smx_tests.log 2>&1; echo "rc=$?" >> gpurun_out/smx_tests.log
timeout 300 python tools/op_times.py asr fp16 8192 20 > gpurun_out/smx_times.txt 2>&1
DJINN_SMX=0 TAG=unfused timeout 300 python tools/op_times.py asr fp16 8192 20 >> gpurun_out/smx_times.txt 2>&1
for r in 1096 2048 4096; do timeout 300 python tools/op_times.py asr fp16 $r 20 | tail -1; DJINN_SMX=0 TAG=unfused timeout 300 python tools/op_times.py asr fp16 $r 20 | tail -1; done >> gpurun_out/smx_times.txt 2>&1

#!/bin/bash
mkdir -p gpurun_out
timeout 300 compute-sanitizer --tool memcheck --print-limit 10 python tools/stem_debug.py fp16 3 > gpurun_out/stem_san.log 2>&1; echo "rc=$?" >> gpurun_out/stem_san.log
timeout 900 python -m pytest tests/test_parity_gpu.py -q -x -k "stem or imc" -p no:cacheprovider > gpurun_out/stem_tests.log 2>&1; echo "rc=$?" >> gpurun_out/stem_tests.log
for s in 1 0; do DJINN_STEM=$s TAG=stem$s timeout 300 python tools/op_times.py imc fp16 1024 20; done > gpurun_out/stem_times.txt 2>&1

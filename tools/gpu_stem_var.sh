#!/bin/bash
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_parity_gpu.py -q -x -k "stem or imc" -p no:cacheprovider > gpurun_out/stem_tests.log 2>&1; echo "rc=$?" >> gpurun_out/stem_tests.log
for s in 2 0 1; do DJINN_STEM=$s TAG=stem$s timeout 300 python tools/op_times.py imc fp16 1024 20 | grep "pack\|conv1\|pool1\|total"; done > gpurun_out/stem_var.txt 2>&1
timeout 600 ncu --set full --import-source on -k regex:stem_conv -c 1 -o gpurun_out/stem_full python tools/op_times.py imc fp16 1024 1 > gpurun_out/stem_ncu.log 2>&1

#!/bin/bash
mkdir -p gpurun_out
for e in 1 0; do for a in face dig; do DJINN_PACK_ROWS=$e TAG=rows$e timeout 300 python tools/op_times.py $a fp16 0 20 | grep "pack\|total"; done; done > gpurun_out/packrows.txt 2>&1
timeout 900 python -m pytest tests/test_parity_gpu.py tests/test_layers_gpu.py -q -x -k "face or dig or gen_b or chunking or host_fed" -p no:cacheprovider >> gpurun_out/packrows.txt 2>&1
timeout 900 python -m pytest tests/test_fullsize_gpu.py -q -x -k "face or dig" -p no:cacheprovider >> gpurun_out/packrows.txt 2>&1

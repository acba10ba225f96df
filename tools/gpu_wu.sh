#!/bin/bash
mkdir -p gpurun_out
for e in 1 0; do DJINN_WINDOW_UNROLL=$e TAG=wu$e timeout 300 python tools/op_times.py dig fp16 1600 20 | grep "pack\|conv1\|total"; DJINN_WINDOW_UNROLL=$e TAG=wu$e timeout 300 python tools/fwd_time.py dig fp16 1600 50; done > gpurun_out/wu.txt 2>&1
timeout 900 python -m pytest tests/test_parity_gpu.py tests/test_serving_gpu.py -q -x -k "dig or chunking or host_fed" -p no:cacheprovider >> gpurun_out/wu.txt 2>&1
timeout 900 python -m pytest tests/test_fullsize_gpu.py -q -x -k "dig" -p no:cacheprovider >> gpurun_out/wu.txt 2>&1

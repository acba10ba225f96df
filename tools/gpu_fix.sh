#!/bin/bash
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_parity_gpu.py tests/test_serving_gpu.py -q -x -p no:cacheprovider > gpurun_out/fix.txt 2>&1
timeout 300 python tools/fwd_time.py pos fp16 1792,4096,65536 50 >> gpurun_out/fix.txt 2>&1

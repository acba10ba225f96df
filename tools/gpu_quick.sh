#!/bin/bash
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_parity_gpu.py -q -x -k "split_k or face or imc" -p no:cacheprovider > gpurun_out/quick_tests.log 2>&1; echo "rc=$?" >> gpurun_out/quick_tests.log
for v in 1 0; do DJINN_SPLITK=$v TAG=sk$v timeout 300 python tools/fwd_time.py imc fp16 16,128 30; DJINN_SPLITK=$v TAG=sk$v timeout 300 python tools/fwd_time.py face fp16 2,32,256 30; DJINN_SPLITK=$v TAG=sk$v timeout 300 python tools/fwd_time.py dig fp16 16 30; done > gpurun_out/quick_times.txt 2>&1

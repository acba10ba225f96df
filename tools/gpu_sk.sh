#!/bin/bash
mkdir -p gpurun_out
for e in 1 0; do
  DJINN_SPLITK_WIDE=$e TAG=wide$e timeout 300 python tools/op_times.py imc fp16 1024 20 | grep "fc\|total"
  DJINN_SPLITK_WIDE=$e TAG=wide$e timeout 300 python tools/op_times.py face fp16 256 20 | grep "F7\|F8\|total"
  DJINN_SPLITK_WIDE=$e TAG=wide$e timeout 300 python tools/fwd_time.py imc fp16 16,128,1024 30
  DJINN_SPLITK_WIDE=$e TAG=wide$e timeout 300 python tools/fwd_time.py face fp16 2,32,256 30
done > gpurun_out/sk.txt 2>&1
timeout 900 python -m pytest tests/test_parity_gpu.py -q -x -k "split or imc or face" -p no:cacheprovider >> gpurun_out/sk.txt 2>&1
timeout 900 python -m pytest tests/test_fullsize_gpu.py -q -x -k "imc or face" -p no:cacheprovider >> gpurun_out/sk.txt 2>&1

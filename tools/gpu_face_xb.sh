#!/bin/bash
mkdir -p gpurun_out
for xb in 8 4; do DJINN_KX_XB=$xb TAG=kxxb$xb timeout 300 python tools/op_times.py face fp16 256 20 | grep "pack\|C1\|total"; done > gpurun_out/face_xb.txt 2>&1
for xb in 8 4; do DJINN_KX_XB=$xb TAG=kxxb$xb timeout 300 python tools/fwd_time.py face fp16 2,32,256 30; done >> gpurun_out/face_xb.txt 2>&1
DJINN_KX_XB=4 timeout 900 python -m pytest tests/test_parity_gpu.py -q -x -k "face" -p no:cacheprovider >> gpurun_out/face_xb.txt 2>&1

#!/bin/bash
mkdir -p gpurun_out
for xb in 8 4 2; do DJINN_LC_XB=$xb TAG=xb$xb timeout 300 python tools/op_times.py face fp16 256 20 | grep " L[456]\|total"; done > gpurun_out/quick_times.txt 2>&1
for xb in 8 4; do DJINN_LC_XB=$xb TAG=xb$xb timeout 300 python tools/fwd_time.py face fp16 2,32,256 30; done >> gpurun_out/quick_times.txt 2>&1

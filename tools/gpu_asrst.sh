#!/bin/bash
mkdir -p gpurun_out
DJINN_LIB=paper_conf_isca_hauswaldklclmdm15_b200/libdjinn_stats.so timeout 300 python tools/op_once.py asr fp16 8192 > gpurun_out/asrst.txt 2>&1
for bn in 0 128 256; do DJINN_DENSE_BN=$bn TAG=bn$bn timeout 300 python tools/op_times.py asr fp16 8192 20 | grep "a0\|a1 \|out\|total"; done >> gpurun_out/asrst.txt 2>&1

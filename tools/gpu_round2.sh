#!/bin/bash
# stats build role timing for DIG, then the full GPU round (tests, smoke, bench)
mkdir -p gpurun_out
DJINN_LIB=paper_conf_isca_hauswaldklclmdm15_b200/libdjinn_stats.so timeout 300 python tools/op_once.py dig fp16 1600 > gpurun_out/dig_stats.txt 2>&1
bash tools/gpu_round.sh

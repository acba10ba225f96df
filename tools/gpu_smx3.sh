#!/bin/bash
mkdir -p gpurun_out
for v in libdjinn.so libdjinn_nomc.so; do DJINN_LIB=paper_conf_isca_hauswaldklclmdm15_b200/$v TAG=$v timeout 300 python tools/op_times.py asr fp16 8192 20 | grep "out\|total"; done > gpurun_out/smx3.txt 2>&1
DJINN_LIB=paper_conf_isca_hauswaldklclmdm15_b200/libdjinn_nomc.so timeout 600 python -m pytest tests/test_fused_gpu.py -x -q -p no:cacheprovider >> gpurun_out/smx3.txt 2>&1

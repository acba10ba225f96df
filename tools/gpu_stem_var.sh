#!/bin/bash
mkdir -p gpurun_out
D=paper_conf_isca_hauswaldklclmdm15_b200
for v in _sc; do DJINN_LIB=$D/libdjinn$v.so TAG=v$v timeout 300 python tools/op_times.py imc fp16 1024 20 | grep "conv1"; done > gpurun_out/stem_var.txt 2>&1
DJINN_LIB=$D/libdjinn_stats.so timeout 120 python tools/op_times.py imc fp16 1024 1 2>&1 | grep "stem\|conv1" > gpurun_out/stats.log

#!/bin/bash
mkdir -p gpurun_out
for sp in 1 4; do DJINN_MLP_SPLIT=$sp DJINN_LIB=paper_conf_isca_hauswaldklclmdm15_b200/libdjinn_mlpstats.so timeout 300 python tools/op_once.py dig fp16 1600; done > gpurun_out/digst.txt 2>&1

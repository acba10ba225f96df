#!/bin/bash
mkdir -p gpurun_out
for v in libdjinn.so libdjinn_nostore.so libdjinn_noepi.so; do DJINN_LIB=paper_conf_isca_hauswaldklclmdm15_b200/$v TAG=$v timeout 300 python tools/op_times.py dig fp16 1600 20 | grep "conv"; DJINN_LIB=paper_conf_isca_hauswaldklclmdm15_b200/$v TAG=$v timeout 300 python tools/op_times.py face fp16 256 20 | grep " C\| L"; done > gpurun_out/xb2.txt 2>&1

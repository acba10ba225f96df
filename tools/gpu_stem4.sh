#!/bin/bash
mkdir -p gpurun_out
for rep in 1 2; do for v in libdjinn.so libdjinn_nwg3.so libdjinn_cb0nwg3.so libdjinn_sf3.so libdjinn_sf4.so libdjinn_cb0sf3.so; do DJINN_LIB=paper_conf_isca_hauswaldklclmdm15_b200/$v TAG=$v timeout 300 python tools/op_times.py imc fp16 1024 20 | grep "conv1"; done; done > gpurun_out/stem4.txt 2>&1

#!/bin/bash
mkdir -p gpurun_out
for rep in 1 2; do for v in libdjinn_prev.so libdjinn.so libdjinn_cb1.so; do DJINN_LIB=paper_conf_isca_hauswaldklclmdm15_b200/$v TAG=$v timeout 300 python tools/op_times.py imc fp16 1024 20 | grep "conv1"; done; done > gpurun_out/stem5.txt 2>&1
timeout 900 python -m pytest tests/test_parity_gpu.py -q -x -k "stem or imc" -p no:cacheprovider >> gpurun_out/stem5.txt 2>&1
timeout 900 python -m pytest tests/test_fullsize_gpu.py -q -x -k "imc" -p no:cacheprovider >> gpurun_out/stem5.txt 2>&1
DJINN_LIB=paper_conf_isca_hauswaldklclmdm15_b200/libdjinn_cb1.so timeout 900 python -m pytest tests/test_parity_gpu.py -q -x -k "stem" -p no:cacheprovider >> gpurun_out/stem5.txt 2>&1

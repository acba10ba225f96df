#!/bin/bash
mkdir -p gpurun_out
for rep in 1 2; do for v in libdjinn.so libdjinn_wk64.so; do DJINN_LIB=paper_conf_isca_hauswaldklclmdm15_b200/$v TAG=$v timeout 300 python tools/fwd_time.py pos fp16 1792,4096,65536 50; done; done > gpurun_out/wk.txt 2>&1
DJINN_LIB=paper_conf_isca_hauswaldklclmdm15_b200/libdjinn_wk64.so timeout 900 python -m pytest tests/test_parity_gpu.py -q -x -k "pos or chk or ner" -p no:cacheprovider >> gpurun_out/wk.txt 2>&1

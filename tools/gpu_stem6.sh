#!/bin/bash
mkdir -p gpurun_out
for v in libdjinn.so libdjinn_cb1pad.so libdjinn_cb0n3.so libdjinn_cb1.so; do
  echo "== $v" ; DJINN_LIB=paper_conf_isca_hauswaldklclmdm15_b200/$v TAG=$v timeout 300 python tools/op_times.py imc fp16 1024 20 | grep "conv1"
  DJINN_LIB=paper_conf_isca_hauswaldklclmdm15_b200/$v timeout 600 python -m pytest tests/test_parity_gpu.py -q -k "stem" -p no:cacheprovider 2>&1 | tail -2
done > gpurun_out/stem6.txt 2>&1

#!/bin/bash
mkdir -p gpurun_out
for v in libdjinn.so libdjinn_cb1pad.so; do
  echo "== $v" ; for rep in 1 2; do DJINN_LIB=paper_conf_isca_hauswaldklclmdm15_b200/$v TAG=$v timeout 300 python tools/op_times.py imc fp16 1024 20 | grep "conv1"; done
  for rep in 1 2 3; do DJINN_LIB=paper_conf_isca_hauswaldklclmdm15_b200/$v timeout 600 python -m pytest tests/test_parity_gpu.py -q -k "stem" -p no:cacheprovider 2>&1 | tail -1; done
  DJINN_LIB=paper_conf_isca_hauswaldklclmdm15_b200/$v timeout 600 python -m pytest tests/test_fullsize_gpu.py -q -k "imc" -p no:cacheprovider 2>&1 | tail -1
done > gpurun_out/stem7.txt 2>&1

#!/bin/bash
mkdir -p gpurun_out
for v in libdjinn.so libdjinn_mlp256.so; do DJINN_LIB=paper_conf_isca_hauswaldklclmdm15_b200/$v TAG=$v timeout 300 python tools/fwd_time.py pos fp16 1792,4096,65536 50; done > gpurun_out/mlp_rpc.txt 2>&1
timeout 300 python tools/fwd_time.py ner fp16 1792,4096,65536 50 >> gpurun_out/mlp_rpc.txt 2>&1
DJINN_LIB=paper_conf_isca_hauswaldklclmdm15_b200/libdjinn_mlpstats.so timeout 300 python tools/op_once.py pos fp16 4096 >> gpurun_out/mlp_rpc.txt 2>&1
timeout 900 python -m pytest tests/test_parity_gpu.py -q -x -k "pos or chk or ner or mlp" -p no:cacheprovider >> gpurun_out/mlp_rpc.txt 2>&1
timeout 900 python -m pytest tests/test_fullsize_gpu.py -q -x -k "pos or chk or ner" -p no:cacheprovider >> gpurun_out/mlp_rpc.txt 2>&1

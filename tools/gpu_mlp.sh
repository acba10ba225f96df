#!/bin/bash
mkdir -p gpurun_out
DJINN_LIB=paper_conf_isca_hauswaldklclmdm15_b200/libdjinn_mst.so python tools/fwd_time.py pos fp16 4096 3 2>&1 | tail -3 > gpurun_out/mst.txt
timeout 900 python -m pytest tests/test_parity_gpu.py -q -x -k "mlp or pos or chk or ner or modes" -p no:cacheprovider > gpurun_out/mlp_tests.log 2>&1; echo "rc=$?" >> gpurun_out/mlp_tests.log
for a in pos ner; do DJINN_MLP=1 TAG=mlp1 timeout 300 python tools/fwd_time.py $a fp16 28,1792,4096,65536,1048576 50; done > gpurun_out/mlp_times.txt 2>&1

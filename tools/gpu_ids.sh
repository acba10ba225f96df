#!/bin/bash
mkdir -p gpurun_out
for m in 1 0; do DJINN_MLP=$m TAG=mlp$m timeout 300 python tools/fwd_time.py pos_ids fp16 1792,4096,65536 50; DJINN_MLP=$m TAG=mlp$m timeout 300 python tools/fwd_time.py ner_ids fp16 4096 50; done > gpurun_out/ids.txt 2>&1
timeout 900 python -m pytest tests/test_parity_gpu.py -q -x -k "token or ids" -p no:cacheprovider >> gpurun_out/ids.txt 2>&1

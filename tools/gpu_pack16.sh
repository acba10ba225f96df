#!/bin/bash
mkdir -p gpurun_out
timeout 300 python tools/op_times.py asr fp16 8192 20 | grep "pack\|total" > gpurun_out/pack16.txt 2>&1
timeout 300 python tools/fwd_time.py asr fp16 1096,8192 30 >> gpurun_out/pack16.txt 2>&1
timeout 900 python -m pytest tests/test_parity_gpu.py tests/test_serving_gpu.py tests/test_layers_gpu.py -q -x -k "asr or pos or chk or ner or concurrent or gen_w or binding" -p no:cacheprovider >> gpurun_out/pack16.txt 2>&1
timeout 900 python -m pytest tests/test_fullsize_gpu.py tests/test_fused_gpu.py -q -x -k "asr or fused or cluster" -p no:cacheprovider >> gpurun_out/pack16.txt 2>&1

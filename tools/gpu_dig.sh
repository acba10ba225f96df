#!/bin/bash
mkdir -p gpurun_out
timeout 300 python tools/op_times.py dig fp16 1600 20 > gpurun_out/dig.txt 2>&1
DJINN_MLP=0 TAG=unfused timeout 300 python tools/op_times.py dig fp16 1600 20 >> gpurun_out/dig.txt 2>&1
timeout 300 python tools/fwd_time.py dig fp16 1600 50 >> gpurun_out/dig.txt 2>&1
DJINN_MLP=0 TAG=unfused timeout 300 python tools/fwd_time.py dig fp16 1600 50 >> gpurun_out/dig.txt 2>&1
timeout 900 python -m pytest tests/test_parity_gpu.py tests/test_layers_gpu.py -q -x -k "dig or mlp or generic or gen_ or lrn_placements" -p no:cacheprovider >> gpurun_out/dig.txt 2>&1
timeout 900 python -m pytest tests/test_fullsize_gpu.py -q -x -k "dig" -p no:cacheprovider >> gpurun_out/dig.txt 2>&1

#!/bin/bash
mkdir -p gpurun_out
for a in dig face imc asr; do timeout 300 python tools/op_times.py $a fp16 0 20; done > gpurun_out/xb.txt 2>&1
timeout 1500 python -m pytest tests/test_parity_gpu.py tests/test_layers_gpu.py tests/test_fullsize_gpu.py -q -x -p no:cacheprovider >> gpurun_out/xb.txt 2>&1

#!/bin/bash
# IMC first-layer kernel study: role timing (stats build), per-op times, ncu of the stem kernel.
mkdir -p gpurun_out
DJINN_LIB=paper_conf_isca_hauswaldklclmdm15_b200/libdjinn_sstats.so timeout 300 python tools/op_once.py imc fp16 1024 > gpurun_out/stem_stats.txt 2>&1
timeout 300 python tools/op_times.py imc fp16 1024 20 > gpurun_out/imc_times.txt 2>&1
timeout 300 python tools/op_times.py dig fp16 1600 20 >> gpurun_out/imc_times.txt 2>&1
timeout 300 python tools/op_times.py face fp16 256 20 >> gpurun_out/imc_times.txt 2>&1
bash tools/gpu_ncu_stem.sh

#!/bin/bash
mkdir -p gpurun_out
export DJINN_PDL=0
export X=1
timeout 300 compute-sanitizer --tool memcheck --print-limit 20 python tools/stem_debug.py fp16 3 > gpurun_out/stem_san.log 2>&1
echo "rc=$?" >> gpurun_out/stem_san.log

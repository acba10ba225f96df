#!/bin/bash
mkdir -p gpurun_out
DJINN_HOST_PROF=1 python tools/host_overhead.py dig fp16 1600 > gpurun_out/host.txt 2>&1
DJINN_HOST_PROF=1 DJINN_MLP=0 python tools/host_overhead.py pos fp16 4096 >> gpurun_out/host.txt 2>&1

#!/bin/bash
mkdir -p gpurun_out
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,power.limit,temperature.gpu --format=csv > gpurun_out/smi.txt 2>&1
for i in 1 2; do timeout 900 python bench.py --steps 20 --warmup 5 > gpurun_out/bench_$i.json 2> gpurun_out/bench_$i.err; done

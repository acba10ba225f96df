#!/bin/bash
mkdir -p gpurun_out
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -c 800 --csv --log-file gpurun_out/launches.csv \
  python bench.py --steps 2 --warmup 3 --headline-only > gpurun_out/launches_bench.log 2>&1
echo "rc=$?" >> gpurun_out/launches_bench.log

#!/bin/bash
mkdir -p gpurun_out /tmp/ncu
timeout 900 ncu --set full --import-source on --clock-control none -k regex:stem_conv -c 1 -o /tmp/ncu/stem -f python tools/op_once.py imc fp16 > gpurun_out/stemprof.log 2>&1
ncu -i /tmp/ncu/stem.ncu-rep --page source --csv --print-source sass > /tmp/ncu/stem_sass.csv 2>/dev/null
python tools/sass_hot.py /tmp/ncu/stem_sass.csv 45 > gpurun_out/stem_hot.txt 2>&1
ncu -i /tmp/ncu/stem.ncu-rep --page details --csv > gpurun_out/stem_details.csv 2>/dev/null

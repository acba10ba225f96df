#!/bin/bash
mkdir -p gpurun_out
for bn in -1 128 192; do
  for a in asr imc; do
    if [ "$bn" = "-1" ]; then unset DJINN_DENSE_BN; else export DJINN_DENSE_BN=$bn; fi
    TAG=bn$bn timeout 300 python tools/op_times.py $a fp16 $([ $a = asr ] && echo 8192 || echo 1024) 20 | grep -E " a[0-9]| out|fc[678]|total"
  done
done > gpurun_out/bn.txt 2>&1

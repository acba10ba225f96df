#!/bin/bash
mkdir -p gpurun_out
DJINN_LIB=paper_conf_isca_hauswaldklclmdm15_b200/libdjinn_smxstats.so timeout 300 python tools/op_once.py asr fp16 8192 > gpurun_out/smx4.txt 2>&1

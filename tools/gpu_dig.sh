#!/bin/bash
mkdir -p gpurun_out
timeout 300 python tools/op_times.py dig fp16 1600 20 > gpurun_out/dig.txt 2>&1
for sp in 1 2 4; do DJINN_MLP_SPLIT=$sp TAG=split$sp timeout 300 python tools/fwd_time.py dig fp16 1600 50 >> gpurun_out/dig.txt 2>&1; done
timeout 900 python -m pytest tests/test_parity_gpu.py tests/test_layers_gpu.py -q -x -k "dig or mlp or generic or gen_" -p no:cacheprovider >> gpurun_out/dig.txt 2>&1
timeout 900 python -m pytest tests/test_fullsize_gpu.py -q -x -k "dig" -p no:cacheprovider >> gpurun_out/dig.txt 2>&1
#!/bin/bash
mkdir -p gpurun_out
for sp in 1 4; do DJINN_MLP_SPLIT=$sp DJINN_LIB=paper_conf_isca_hauswaldklclmdm15_b200/libdjinn_mlpstats.so timeout 300 python tools/op_once.py dig fp16 1600; done > gpurun_out/digst.txt 2>&1

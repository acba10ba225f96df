# IMC first layer: fused pool (DJINN_STEM=3) vs TMA-store stem + pool (2); bitwise tests vs the generic path.
mkdir -p gpurun_out
{ for v in 3 2; do DJINN_STEM=$v TAG=stem$v timeout 300 python tools/op_times.py imc fp16 1024 10 2>&1 | grep -E "conv1|pool1|pack|total"; done;
  for n in 16 128; do DJINN_STEM=3 TAG=stem3-$n timeout 300 python tools/op_times.py imc fp16 $n 20 2>&1 | grep -E "conv1|pool1|total"; 
  DJINN_STEM=2 TAG=stem2-$n timeout 300 python tools/op_times.py imc fp16 $n 20 2>&1 | grep -E "conv1|pool1|total"; done; } > gpurun_out/stempool.txt 2>&1
timeout 1200 python -m pytest tests/test_parity_gpu.py -m gpu -q -x --timeout 600 -k "stem and 3" > gpurun_out/pytest_stem.log 2>&1; tail -3 gpurun_out/pytest_stem.log
cat gpurun_out/stempool.txt

# PDL / new s2d pack correctness, loader-wait policy sweep, LRN MUFU-count diagnostics
mkdir -p gpurun_out
L=$PWD/paper_conf_isca_hauswaldklclmdm15_b200
timeout 900 python -m pytest tests -m gpu -q -x --timeout 600 > gpurun_out/pytest_gpu.log 2>&1; tail -3 gpurun_out/pytest_gpu.log
for w in 0 1 2; do for a in imc face; do DJINN_LDWAIT=$w TAG=ldwait$w timeout 300 python tools/op_times.py $a bf16 2>&1 | grep -E "conv|C1|pack|total"; done; done
for v in lrn0 lrn1; do DJINN_LIB=$L/libdjinn_$v.so TAG=$v timeout 300 python tools/op_times.py imc bf16 2>&1 | grep -E "conv1|conv2"; done
for p in 0 1; do DJINN_PDL=$p timeout 600 python bench.py --steps 30 --no-cpu-baseline --no-e2e > gpurun_out/bench_pdl$p.json 2>&1; python -c "
import json;d=json.loads(open('gpurun_out/bench_pdl$p.json').read().strip().splitlines()[-1]);print('PDL=$p', d['ms_per_step'], {a:round(v['ms_per_batch'],3) for a,v in d['per_app'].items()})"; done

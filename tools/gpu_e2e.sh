# Host-fed pipeline check: its parity tests, then the bench at several pipeline depths / service modes.
set -u
mkdir -p gpurun_out
timeout 600 python -m pytest tests/test_parity_gpu.py -q -rf -k "host" > gpurun_out/pytest_e2e.log 2>&1; tail -3 gpurun_out/pytest_e2e.log
for sv in ${SERVICES:-concurrent serial}; do
for c in ${CHUNKS:-1 2 4}; do
  DJINN_PIPE_CHUNKS=$c timeout 600 python bench.py --steps 20 --no-cpu-baseline --services $sv > gpurun_out/bench_e2e_${sv}_$c.json 2> gpurun_out/bench_e2e_${sv}_$c.err
  python -c "import json,sys;d=json.loads(open('gpurun_out/bench_e2e_${sv}_$c.json').read().strip().splitlines()[-1]);print('$sv chunks $c', round(d['ms_per_step'],3), round(d['e2e']['ms_per_step'],3), d['roofline']['avg_us_in_timed_region'])"
done; done

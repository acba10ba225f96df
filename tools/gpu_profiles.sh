#!/bin/bash
# ncu captures of every kernel of each app's forward (fp16, bench batch) summarised on the box
# (reports are too large to bring back), the bench launch list, compute-sanitizer on small shapes.
mkdir -p gpurun_out /tmp/ncu
for a in imc face asr dig pos; do
  timeout 900 ncu --set full --clock-control none -o /tmp/ncu/ncu_$a -f python tools/op_once.py $a fp16 > gpurun_out/ncu_$a.log 2>&1
  python tools/ncu_summary.py /tmp/ncu/ncu_$a.ncu-rep $a gpurun_out/ncu_$a.log >> gpurun_out/ncu_kernels.jsonl 2>> gpurun_out/ncu_summary.err
done
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -c 800 --csv --log-file gpurun_out/launches.csv \
  python bench.py --steps 2 --warmup 3 --headline-only > gpurun_out/launches_bench.log 2>&1
for t in memcheck racecheck synccheck; do
  timeout 1200 compute-sanitizer --tool $t --print-limit 20 python tools/sanitize_small.py > gpurun_out/san_$t.log 2>&1
  echo "rc=$?" >> gpurun_out/san_$t.log
done

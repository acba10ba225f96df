# ncu --set full of the IMC first-layer kernel (fused pool) + SASS stall summary and pipe metrics.
mkdir -p gpurun_out /tmp/ncu
timeout 900 ncu --set full --clock-control none --import-source on -k regex:stem_conv -c 1 -o /tmp/ncu/stem -f python tools/op_once.py imc fp16 1024 > gpurun_out/ncu_stem.log 2>&1
ncu -i /tmp/ncu/stem.ncu-rep --page source --csv --print-source sass > /tmp/ncu/stem_src.csv 2>/dev/null
python tools/ncu_stalls.py /tmp/ncu/stem_src.csv 40 > gpurun_out/stem_stalls.txt 2>&1
ncu -i /tmp/ncu/stem.ncu-rep --page raw --csv > /tmp/ncu/stem_raw.csv 2>/dev/null
python - > gpurun_out/stem_metrics.txt <<'PY'
import csv
rows=list(csv.reader(open('/tmp/ncu/stem_raw.csv')))
h,u,r=rows[0],rows[1],rows[2]
keys=['gpu__time_duration.sum','sm__inst_issued.avg.pct_of_peak_sustained_active','sm__pipe_tensor_cycles_active.avg.pct_of_peak_sustained_elapsed',
'dram__bytes_read.sum','dram__bytes_write.sum','smsp__inst_executed.sum','sm__warps_active.avg.pct_of_peak_sustained_active']
for i,k in enumerate(h):
    if k in keys or 'pipe_xu' in k or 'pipe_fma' in k or 'pipe_alu' in k or 'warp_issue_stalled' in k and 'pct' in k or 'pipe_uniform' in k or 'pipe_lsu' in k or 'inst_executed_pipe' in k:
        print(k, u[i], r[i])
PY
tail -3 gpurun_out/ncu_stem.log

#!/bin/bash
mkdir -p gpurun_out /tmp/ncu
./tools/cluster_occ > gpurun_out/cluster_occ.txt 2>&1
timeout 600 ncu --set full --clock-control none -k regex:smx_kernel -c 1 -o /tmp/ncu/smx -f python tools/op_once.py asr fp16 8192 > gpurun_out/ncu_smx.log 2>&1
ncu -i /tmp/ncu/smx.ncu-rep --page raw --csv > /tmp/ncu/smx_raw.csv 2>/dev/null
python - > gpurun_out/smx_metrics.txt <<'PY'
import csv
rows=list(csv.reader(open('/tmp/ncu/smx_raw.csv')))
h,u,r=rows[0],rows[1],rows[2]
for i,k in enumerate(h):
    if any(x in k for x in ('gpu__time_duration.sum','sm__pipe_tensor_cycles_active.avg.pct','dram__bytes_read.sum','dram__bytes_write.sum',
       'lts__t_bytes.sum','sm__warps_active.avg.pct','launch__cluster','launch__grid_size','sm__cycles_active.avg','lts__throughput.avg.pct',
       'l1tex__m_xbar2l1tex_read_bytes.sum','sm__throughput.avg.pct','launch__occupancy_cluster','smsp__warp_issue_stalled')) and not k.endswith('per_second'):
        print(k, u[i], r[i])
PY

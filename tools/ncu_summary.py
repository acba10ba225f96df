"""Per-kernel summary of an `ncu --set full` report of tools/op_once.py (run where the report
is; writes one JSON line per kernel launch).  usage: python tools/ncu_summary.py REP APP LOG"""
import csv
import json
import subprocess
import sys

rep, app, log = sys.argv[1], sys.argv[2], sys.argv[3]
order = []
for ln in open(log):
    if ln.startswith("LAUNCH_ORDER"):
        order = ln.split()[1:]
M = {"dur": "gpu__time_duration.sum", "dram_rd": "dram__bytes_read.sum", "dram_wr": "dram__bytes_write.sum",
     "tensor_pct": "sm__pipe_tensor_cycles_active.avg.pct_of_peak_sustained_elapsed",
     "sm_pct": "sm__throughput.avg.pct_of_peak_sustained_elapsed",
     "dram_pct": "gpu__dram_throughput.avg.pct_of_peak_sustained_elapsed",
     "l2_hit": "lts__t_sector_hit_rate.pct", "issue_pct": "sm__inst_issued.avg.pct_of_peak_sustained_active",
     "regs": "launch__registers_per_thread", "grid": "launch__grid_size"}
raw = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
rows = list(csv.reader(raw.splitlines()))
h, u = rows[0], rows[1]
scale = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9, "nsecond": 1e-3, "usecond": 1.0, "msecond": 1e3}
ki = h.index("Kernel Name")
for i, r in enumerate(rows[2:]):
    d = {"app": app, "launch": i, "op": order[i] if i < len(order) else "?", "kernel": r[ki].split("(")[0][:90]}
    for k, m in M.items():
        if m in h:
            j = h.index(m)
            try:
                v = float(r[j].replace(",", ""))
            except ValueError:
                continue
            if k in ("dur", "dram_rd", "dram_wr"):
                v *= scale.get(u[j], 1.0)
            d[k] = v
    if "dur" in d:
        d["dur_us"] = d.pop("dur")
    print(json.dumps(d))

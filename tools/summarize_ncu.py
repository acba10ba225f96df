"""Summarise ncu outputs into profiles/:  launch list (per-kernel device-time shares of the
bench command) and DRAM traffic of the top kernel's full capture (profiles/traffic.json)."""
import csv
import json
import os
import subprocess
import sys
from collections import OrderedDict, defaultdict

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def launches(csv_path, out_md, tag):
    rows = [r for r in csv.reader(open(csv_path)) if r]
    hi = next(i for i, r in enumerate(rows) if "Kernel Name" in r)
    h = rows[hi]
    ki, mi, vi = h.index("Kernel Name"), h.index("Metric Name"), h.index("Metric Value")
    agg = defaultdict(lambda: [0, 0.0])
    total = 0.0
    for r in rows[hi + 1:]:
        if len(r) != len(h) or r[mi] != "gpu__time_duration.sum":
            continue
        name = r[ki].split("(")[0].replace("void ", "").replace("djinn::", "").replace("(anonymous namespace)::", "")
        v = float(r[vi].replace(",", ""))
        agg[name][0] += 1
        agg[name][1] += v
        total += v
    unit = rows[hi + 1][h.index("Metric Unit")] if "Metric Unit" in h else "ns"
    with open(out_md, "w") as f:
        f.write(f"# {tag}: ncu launch list of `bench.py --steps 2 --warmup 3` (gpu__time_duration.sum, "
                f"--clock-control none; cold-cache, serialised: compare SHARES)\n\n")
        f.write(f"| kernel | launches | total ({unit}) | share |\n|---|---|---|---|\n")
        for k, (n, t) in sorted(agg.items(), key=lambda kv: -kv[1][1]):
            f.write(f"| `{k}` | {n} | {t:.0f} | {100 * t / total:.1f}% |\n")
    print(open(out_md).read())


def traffic(rep, key, out_json):
    raw = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
    rows = list(csv.reader(raw.splitlines()))
    h, u = rows[0], rows[1]
    d = OrderedDict()
    for k in ("gpu__time_duration.sum", "dram__bytes_read.sum", "dram__bytes_write.sum",
              "sm__pipe_tensor_cycles_active.avg.pct_of_peak_sustained_elapsed", "lts__t_bytes.sum",
              "sm__throughput.avg.pct_of_peak_sustained_elapsed", "launch__grid_size", "launch__registers_per_thread"):
        if k in h:
            d[k] = (rows[2][h.index(k)], u[h.index(k)])
    scale = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9}
    dram = sum(float(d[k][0].replace(",", "")) * scale.get(d[k][1], 1) for k in ("dram__bytes_read.sum", "dram__bytes_write.sum"))
    out = json.load(open(out_json)) if os.path.exists(out_json) else {}
    out[key] = {"dram_bytes_per_launch": dram, "source": os.path.basename(rep), "metrics": d}
    json.dump(out, open(out_json, "w"), indent=1)
    print(json.dumps(out[key], indent=1))


if __name__ == "__main__":
    cmd = sys.argv[1]
    if cmd == "launches":
        launches(sys.argv[2], sys.argv[3], sys.argv[4])
    else:
        traffic(sys.argv[2], sys.argv[3], sys.argv[4])

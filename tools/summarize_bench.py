"""Write profiles/<tag>_bench_line.json and <tag>_bench_summary.md from a bench.py JSON line.

usage: python tools/summarize_bench.py gpurun_out/bench.json r01
"""
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
src, tag = sys.argv[1], sys.argv[2]
d = json.loads(open(src).read().strip().splitlines()[-1])
with open(os.path.join(ROOT, "profiles", f"{tag}_bench_line.json"), "w") as f:
    f.write(json.dumps(d) + "\n")
r = d["roofline"]
L = [f"# {tag} bench summary (bench.py default run on {d['n_gpus']} x B200)\n",
     f"value {d['value']:.0f} mixed queries/s, {d['ms_per_step']:.3f} ms/step, dtype {d['dtype']}, "
     f"launches {d['gpu_launches']} ({d['gpu_launches'] / d['steps']:.0f}/step), clocks {d['clocks']}\n",
     f"e2e (pinned host buffers): {d['e2e']['value']:.0f} q/s, {d['e2e']['ms_per_step']:.2f} ms/step\n" if d.get("e2e") else "",
     (f"concurrent services (one stream per app): {d['concurrent_services']['value']:.0f} q/s, "
      f"{d['concurrent_services']['ms_per_step']:.3f} ms/step"
      + (f"; host-fed {d['concurrent_services']['e2e']['ms_per_step']:.2f} ms/step" if d['concurrent_services'].get('e2e') else "")
      + "\n") if d.get("concurrent_services") else "",
     f"cpu_baseline (fp64 oracle, {d['cpu_baseline']['cores']} threads): {d['cpu_baseline']['value']:.2f} q/s\n"
     if d.get("cpu_baseline") else "",
     f"roofline: {json.dumps(r)}\n",
     "| app | queries/s | ms/batch | roofline ms | frac |", "|---|---|---|---|---|"]
for a, v in d["per_app"].items():
    L.append(f"| {a} | {v['queries_per_s']:.0f} | {v['ms_per_batch']:.3f} | {v['roofline_ms']:.3f} | {v['roofline_frac']:.3f} |")
if any("host_fed" in v for v in d["per_app"].values()):
    L += ["", "host-fed (pinned H2D + D2H per batch, one app alone):", "",
          "| app | queries/s | ms/batch | bytes/query | PCIe GB/s achieved | GB/s needed at device rate |",
          "|---|---|---|---|---|---|"]
    for a, v in d["per_app"].items():
        h = v.get("host_fed")
        if h:
            L.append(f"| {a} | {h['queries_per_s']:.0f} | {h['ms_per_batch']:.3f} | {h['bytes_per_query']:.0f} | "
                     f"{h['pcie_gbs_achieved']:.1f} | {h['pcie_gbs_needed_at_device_rate']:.0f} |")
L += ["", "| app/op | kind | avg us | roofline us | TF/s | GB/s | bound |", "|---|---|---|---|---|---|---|"]
for o in d["top_ops"]:
    L.append(f"| {o['app']}/{o['op']} | {o['kind']} | {o['avg_us']:.1f} | {o['roofline_us']:.1f} | {o['tflops']:.1f} | "
             f"{o['gbs']:.0f} | {o['bound']} |")
with open(os.path.join(ROOT, "profiles", f"{tag}_bench_summary.md"), "w") as f:
    f.write("\n".join(L) + "\n")
print("\n".join(L))

"""profiles/<tag>_ncu_kernels.md and profiles/traffic.json from the per-kernel ncu summaries
(gpurun_out/ncu_kernels.jsonl, written on the GPU box by tools/ncu_summary.py).

usage: python tools/ncu_table.py gpurun_out/ncu_kernels.jsonl r02 "<source note>"
"""
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
src, tag, note = sys.argv[1], sys.argv[2], sys.argv[3] if len(sys.argv) > 3 else ""
recs = [json.loads(l) for l in open(src) if l.strip()]
lines = [f"# {tag}: ncu `--set full --clock-control none` of every kernel of one fp16 forward per app (bench batch)", "",
         "Cold cache, one launch each, clocks not locked (`tools/gpu_profiles.sh`, summarised on the box by "
         "`tools/ncu_summary.py`, tabulated by `tools/ncu_table.py`). dram = read + write bytes of the launch; tensor = "
         "`sm__pipe_tensor_cycles_active` % of peak; issue = `sm__inst_issued` % of peak; sm = `sm__throughput` %; "
         "dram% = `gpu__dram_throughput` %; l2 hit = `lts__t_sector_hit_rate`." + (" " + note if note else ""), "",
         "| app | op | kernel | us | dram MB | tensor % | issue % | sm % | dram % | l2 hit % | regs |",
         "|---|---|---|---|---|---|---|---|---|---|---|"]
tpath = os.path.join(ROOT, "profiles", "traffic.json")
traffic = json.load(open(tpath)) if os.path.exists(tpath) else {}
for r in recs:
    k = r["kernel"].replace("void ", "")
    mb = (r["dram_rd"] + r["dram_wr"]) / 1e6
    lines.append(f"| {r['app']} | {r['op']} | `{k}` | {r['dur_us']:.1f} | {mb:.1f} | {r['tensor_pct']:.1f} | "
                 f"{r.get('issue_pct', 0):.1f} | {r['sm_pct']:.1f} | {r['dram_pct']:.1f} | {r['l2_hit']:.1f} | {int(r['regs'])} |")
    traffic[f"{r['app']}/{r['op']}"] = {"dram_bytes_per_launch": r["dram_rd"] + r["dram_wr"],
                                       "source": f"{tag} ncu --set full (tools/gpu_profiles.sh)", "duration_us": r["dur_us"],
                                       "tensor_pct": r["tensor_pct"], "sm_pct": r["sm_pct"], "dram_pct": r["dram_pct"],
                                       "l2_hit_pct": r["l2_hit"], "kernel": k}
open(os.path.join(ROOT, "profiles", f"{tag}_ncu_kernels.md"), "w").write("\n".join(lines) + "\n")
json.dump(traffic, open(tpath, "w"), indent=1)
print(len(recs), "kernels")

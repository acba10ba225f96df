"""Device time of whole forward passes (CUDA events around K back-to-back calls, no per-op
profiling).  usage: python tools/fwd_time.py APP PREC ROWS[,ROWS...] [K]"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import paper_conf_isca_hauswaldklclmdm15_b200 as dj  # noqa: E402
from datagen import recipes  # noqa: E402

app, prec = sys.argv[1], sys.argv[2]
rows_list = [int(r) for r in sys.argv[3].split(",")]
K = int(sys.argv[4]) if len(sys.argv) > 4 else 50
tag = os.environ.get("TAG", "")
w = recipes.flat_blob(recipes.gen_weights(app, prec))
base = torch.from_numpy(recipes.gen_input_rows(app, 0, min(max(rows_list), 8192), prec)).cuda()
for rows in rows_list:
    net = dj.DjinnNet(dj.net_description(app), w, prec, rows)
    reps = (rows + base.shape[0] - 1) // base.shape[0]
    x = base.repeat((reps,) + (1,) * (base.dim() - 1))[:rows].contiguous()
    out = torch.empty(rows, net.out_elems, device="cuda")
    s = torch.cuda.Stream()
    for _ in range(5):
        dj.djinn_forward(net.handle, x, rows, out, dj.DJINN_OUT_PROB, s.cuda_stream)
    torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record(s)
    for _ in range(K):
        dj.djinn_forward(net.handle, x, rows, out, dj.DJINN_OUT_PROB, s.cuda_stream)
    e1.record(s)
    torch.cuda.synchronize()
    us = e0.elapsed_time(e1) * 1e3 / K
    print(f"[{tag}] {app} {prec} rows={rows} {us:9.2f} us/batch  {rows / us * 1e6 / 28:12.0f} q/s(28 rows/q)")
    net.close()

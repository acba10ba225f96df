"""Run one Tonic app's forward pass a few times (for ncu / compute-sanitizer captures).

usage: python tools/run_app.py APP [PREC] [ROWS] [ITERS]
"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import paper_conf_isca_hauswaldklclmdm15_b200 as dj  # noqa: E402
from datagen import recipes  # noqa: E402

app = sys.argv[1]
prec = sys.argv[2] if len(sys.argv) > 2 else "bf16"
rows = int(sys.argv[3]) if len(sys.argv) > 3 else {"imc": 1024, "face": 256, "asr": 8192, "dig": 1600}.get(app, 4096)
iters = int(sys.argv[4]) if len(sys.argv) > 4 else 2
net = dj.DjinnNet(dj.net_description(app), recipes.flat_blob(recipes.gen_weights(app, prec)), prec, rows)
x = torch.from_numpy(recipes.gen_input_rows(app, 0, rows, prec)).cuda()
out = torch.empty(rows, net.out_elems, device="cuda")
print(net.plan())
for _ in range(iters):
    net.forward(x, dj.DJINN_OUT_PROB, out=out)
torch.cuda.synchronize()
print("ok", out[:2, :4].tolist())

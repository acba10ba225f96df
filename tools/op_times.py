"""Per-op device times of one Tonic app (CUDA events around every kernel, djinn_profile).

usage: python tools/op_times.py APP [PREC] [ROWS] [ITERS]     (DJINN_LIB selects a variant build)
"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import paper_conf_isca_hauswaldklclmdm15_b200 as dj  # noqa: E402
from datagen import recipes  # noqa: E402

app = sys.argv[1]
prec = sys.argv[2] if len(sys.argv) > 2 else "bf16"
rows = int(sys.argv[3]) if len(sys.argv) > 3 and int(sys.argv[3]) > 0 else {"imc": 1024, "face": 256, "asr": 8192, "dig": 1600}.get(app, 4096)
iters = int(sys.argv[4]) if len(sys.argv) > 4 else 10
net = dj.DjinnNet(dj.net_description(app), recipes.flat_blob(recipes.gen_weights(app, prec)), prec, rows)
x = torch.from_numpy(recipes.gen_input_rows(app, 0, rows, prec)).cuda()
out = torch.empty(rows, net.out_elems, device="cuda")
for _ in range(3):
    net.forward(x, dj.DJINN_OUT_PROB, out=out)
torch.cuda.synchronize()
dj.djinn_profile(net.handle, True)
for _ in range(iters):
    net.forward(x, dj.DJINN_OUT_PROB, out=out)
torch.cuda.synchronize()
prof = dj.djinn_profile_read(net.handle, reset=True)
tot = 0.0
tag = os.environ.get("TAG", os.path.basename(os.environ.get("DJINN_LIB", "libdjinn.so")))
for i, (t, c) in enumerate(prof):
    if c:
        info = dj.djinn_op_info(net.handle, i)
        tot += t / c
        print(f"[{tag}] {app} {info['name']:20s} {info['kind']:8s} {t / c * 1e3:9.1f} us")
print(f"[{tag}] {app} total {tot * 1e3:9.1f} us")

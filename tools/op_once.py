"""One forward pass of one app (for ncu captures of every kernel of the path).
usage: python tools/op_once.py APP PREC [ROWS]"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import paper_conf_isca_hauswaldklclmdm15_b200 as dj  # noqa: E402
from datagen import recipes  # noqa: E402

app, prec = sys.argv[1], sys.argv[2]
rows = int(sys.argv[3]) if len(sys.argv) > 3 else {"imc": 1024, "face": 256, "asr": 8192, "dig": 1600}.get(app, 4096)
net = dj.DjinnNet(dj.net_description(app), recipes.flat_blob(recipes.gen_weights(app, prec)), prec, rows)
x = torch.from_numpy(recipes.gen_input_rows(app, 0, rows, prec)).cuda()
out = net.forward(x, dj.DJINN_OUT_PROB)
torch.cuda.synchronize()
# the ops that launch a kernel, in launch order (fused ops do not launch)
launched = [ln.split()[1] for ln in net.plan().splitlines()[1:] if ln.strip() and "[fused" not in ln]
print("LAUNCH_ORDER " + " ".join(launched))

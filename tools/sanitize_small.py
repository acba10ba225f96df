"""Small forward passes of every kernel family (for compute-sanitizer memcheck / racecheck /
synccheck): every Tonic app in fp16 at a few rows (ragged tiles), IMC in bf16 and fp32, the
first-layer kernel in both modes, the window-MLP kernel and the batcher."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402
import torch  # noqa: E402

import paper_conf_isca_hauswaldklclmdm15_b200 as dj  # noqa: E402
from datagen import recipes  # noqa: E402

cases = [("imc", "fp16", 3), ("imc", "bf16", 2), ("face", "fp16", 2), ("asr", "fp16", 130), ("dig", "fp16", 130),
         ("pos", "fp16", 130), ("ner", "bf16", 70), ("pos_ids", "fp16", 50), ("dig", "fp32", 20)]
if os.environ.get("SAN_QUICK"):
    cases = cases[:2]
for app, prec, n in cases:
    net = dj.DjinnNet(dj.net_description(app), recipes.flat_blob(recipes.gen_weights(app, prec)), prec, n)
    x = torch.from_numpy(recipes.gen_input_rows(app, 0, n, prec)).cuda()
    for mode in (dj.DJINN_OUT_PROB, dj.DJINN_OUT_ARGMAX):
        net.forward(x, mode)
    if app == "pos":
        b = dj.DjinnBatcher(net, n, max_wait_us=0)
        o = np.empty((28, net.out_elems), np.float32)
        b.wait(b.submit(np.ascontiguousarray(x[:28].cpu().numpy()), o))
        b.close()
    net.close()
    print("ok", app, prec, n, flush=True)

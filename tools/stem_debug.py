"""Run IMC conv1 (fused stem) on a few images; used under compute-sanitizer."""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import paper_conf_isca_hauswaldklclmdm15_b200 as dj
from datagen import recipes
prec = sys.argv[1] if len(sys.argv) > 1 else "fp16"
n = int(sys.argv[2]) if len(sys.argv) > 2 else 3
net = dj.DjinnNet(dj.net_description("imc"), recipes.flat_blob(recipes.gen_weights("imc", prec)), prec, n)
print(net.plan())
x = torch.from_numpy(recipes.gen_input_rows("imc", 0, n, prec)).cuda()
dj.djinn_profile(net.handle, True, 1)
out = net.forward(x, dj.DJINN_OUT_LOGITS)
print(out[:, :5])

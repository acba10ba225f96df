"""Parity at BASELINE.json's full sizes in the launch configuration bench.py times (-m gpu):
the whole batch runs on the GPU; sampled rows (first, middle, last, spread) are checked one
by one against the oracle, and properties that hold at any size are checked on every row."""
import numpy as np
import pytest
import torch

import paper_conf_isca_hauswaldklclmdm15_b200 as dj
from datagen import recipes

from parity import REL_LOGIT_TOL, blob, compare_16bit, oracle_rows

pytestmark = pytest.mark.gpu

# bench.py batch (rows) per app and the sampled rows checked against the oracle
FULL = {"imc": 1024, "face": 256, "asr": 8192, "pos": 4096, "chk": 4096, "ner": 4096, "dig": 1600}
SAMPLE = {"imc": 6, "face": 6, "asr": 48, "pos": 400, "chk": 400, "ner": 400, "dig": 120}


@pytest.mark.parametrize("prec", ["bf16", "fp16"])
@pytest.mark.parametrize("app", list(FULL))
def test_full_batch_sampled_parity_and_properties(app, prec):
    n = FULL[app]
    x = recipes.gen_input_rows(app, 0, n, prec)
    net = dj.DjinnNet(dj.net_description(app), blob(app, prec), prec, n)
    xt = torch.from_numpy(x).cuda()
    lg = net.forward(xt, dj.DJINN_OUT_LOGITS)
    pr = net.forward(xt, dj.DJINN_OUT_PROB)
    am = net.forward(xt, dj.DJINN_OUT_ARGMAX)
    net.close()
    # properties on every row
    assert torch.isfinite(lg).all() and torch.isfinite(pr).all()
    torch.testing.assert_close(pr.sum(1), torch.ones(n, device=pr.device), rtol=0, atol=1e-5)
    assert torch.equal(am.long(), lg.argmax(1))
    # sampled rows vs the oracle: first, last, and an even spread (several tiles apart)
    idx = np.unique(np.concatenate([[0, n - 1], np.linspace(0, n - 1, SAMPLE[app]).astype(int)]))
    lg_ref, _ = oracle_rows(app, x[idx], prec)
    r = compare_16bit(lg.cpu().numpy()[idx], lg_ref)
    print(app, prec, "full batch", n, r)
    assert r["rel_max"] <= REL_LOGIT_TOL, r

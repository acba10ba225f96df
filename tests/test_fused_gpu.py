"""GPU parity of the fused-kernel variants added for SURVEY.md 8(f) f4 (-m gpu).

* dense + softmax over a thread-block cluster (k_smx.cu): the last dense layer of a net whose
  output is a wide softmax (ASR: 8000 senones, Table 3) writes the probabilities
  (or the argmax, or the logits) straight from tensor memory.  Checked against the fp64 oracle
  on a generic wide net (N = 5000: 16 CTAs of 320 columns, the last one ragged; K = 300 padded
  to 320; 300 rows = 3 row blocks with a ragged tail), and against the unfused path
  (tc GEMM + softmax kernel, the default) on ASR itself, in every output mode.  The kernel is
  opt-in (DJINN_SMX=1): it is correct but slower than the unfused pair on B200.
"""
import os

import numpy as np
import pytest
import torch

import paper_conf_isca_hauswaldklclmdm15_b200 as dj
from datagen import recipes

import test_layers_gpu as tl
from parity import ELEM_TOL, REL_LOGIT_TOL, blob, compare_16bit

pytestmark = pytest.mark.gpu

GEN_W = """
name: "gen_w"
layer { name: "data" type: "Input" top: "data" input_param { shape { dim: 200 } } }
layer { name: "f1" type: "InnerProduct" bottom: "data" top: "f1" inner_product_param { num_output: 300 } }
layer { name: "r1" type: "ReLU" bottom: "f1" top: "f1" }
layer { name: "f2" type: "InnerProduct" bottom: "f1" top: "f2" inner_product_param { num_output: 5000 } }
layer { name: "prob" type: "Softmax" bottom: "f2" top: "prob" }
"""
tl.NETS.setdefault("gen_w", GEN_W)


def _with_env(env, fn):
    old = {k: os.environ.get(k) for k in env}
    os.environ.update(env)
    try:
        return fn()
    finally:
        for k, v in old.items():
            if v is None:
                os.environ.pop(k, None)
            else:
                os.environ[k] = v


def _forward_all(text, W, x, prec, env):
    def run():
        net = dj.DjinnNet(text, recipes.flat_blob(W) if isinstance(W, list) else W, prec, x.shape[0])
        xt = torch.from_numpy(x).cuda()
        lg = net.forward(xt, dj.DJINN_OUT_LOGITS).cpu().numpy()
        pr = net.forward(xt, dj.DJINN_OUT_PROB).cpu().numpy()
        am = net.forward(xt, dj.DJINN_OUT_ARGMAX).cpu().numpy()
        plan = net.plan()
        net.close()
        return lg, pr, am, plan
    return _with_env(env, run)


@pytest.mark.parametrize("prec", ["fp16", "bf16"])
def test_cluster_softmax_wide_layer_matches_oracle(prec):
    net, W, x = tl.gen_net("gen_w", prec)
    lg_ref, pr_ref = net.forward(x, W)
    lg, pr, am, plan = _forward_all(GEN_W, W, x, prec, {"DJINN_SMX": "1", "DJINN_SMX_MIN_ROWS": "128"})
    print(plan)
    assert "cluster kernel, 16 CTAs x 320 columns" in plan
    r = compare_16bit(lg, lg_ref)
    print(prec, r)
    assert r["rel_max"] <= REL_LOGIT_TOL and r["elem_max"] <= ELEM_TOL, r
    assert r["top1_decidable"] >= 0.99, r
    # probabilities: the softmax of the returned logits (fp64), rows sum to 1; argmax mode is
    # the first maximum of the logits
    z = lg.astype(np.float64)
    p64 = np.exp(z - z.max(1, keepdims=True))
    p64 /= p64.sum(1, keepdims=True)
    assert np.abs(pr - p64).max() <= 1e-6 + 1e-5 * p64.max(), np.abs(pr - p64).max()
    np.testing.assert_allclose(pr.sum(1), 1.0, atol=1e-5)
    assert np.array_equal(am.astype(np.int64), lg.argmax(1))


@pytest.mark.parametrize("rows", [1100, 2048])
def test_cluster_softmax_equals_unfused_asr(rows):
    prec = "fp16"
    W = blob("asr", prec)
    x = recipes.gen_input_rows("asr", 0, rows, prec)
    lg, pr, am, plan = _forward_all(dj.net_description("asr"), W, x, prec, {"DJINN_SMX": "1"})
    lg0, pr0, am0, plan0 = _forward_all(dj.net_description("asr"), W, x, prec, {})
    assert "cluster kernel" in plan and "cluster kernel" not in plan0
    # the same fp32 accumulators + bias: logits agree to fp32 rounding of the MMA order
    d = np.abs(lg - lg0).max() / np.abs(lg0).max()
    print("rows", rows, "logit max rel diff", d, "bitwise", np.array_equal(lg, lg0))
    assert d <= 1e-6
    assert np.abs(pr - pr0).max() <= 1e-6 + 1e-5 * pr0.max()
    assert np.array_equal(am.astype(np.int64), lg.argmax(1))
    assert (am == am0).mean() >= 0.999

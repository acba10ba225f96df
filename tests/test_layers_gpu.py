"""GPU parity of the layer modes the Tonic nets do not use, on small generic nets (-m gpu).

PAPER.md L78 (sec 3.1): DjiNN runs Caffe's configurable layer framework, so djinn.h promises
any description built from its layer set, not only the seven Tonic nets.  These nets
exercise, through the C ABI and against the fp64 oracle: a padded strided first conv (im2col
TMA), LRN (in the conv epilogue, in the lrn+pool kernel and as the standalone kernel), MAX
pooling with pad, a 4-group conv, a locally-connected layer with TanH, AVE pooling with and
without pad (Caffe divisor, reading R10), Sigmoid + Dropout, HardTanh and TanH in dense
epilogues.  Also: a net loaded with weights=NULL whose arena is filled by a device copy from a
loaded net (the C1 broadcast path) reproduces it bitwise, the host-fed staging slots survive
an unsynchronised djinn_forward16 -> djinn_forward sequence, and the binding rejects buffers
the C ABI would read or write out of bounds.
"""
import os
import subprocess
import sys

import numpy as np
import pytest
import torch

import paper_conf_isca_hauswaldklclmdm15_b200 as dj
from paper_conf_isca_hauswaldklclmdm15_b200 import parallel
from datagen import recipes, rng
from oracle import OracleNet

from parity import (ELEM_TOL, FP32_PROB_TOL, REL_LOGIT_TOL, blob, compare_16bit, compare_fp32)

pytestmark = pytest.mark.gpu

# conv(pad, stride) -> LRN -> MAX pool(pad) -> 4-group conv -> LC + TanH -> AVE pool(pad)
# -> IP + Sigmoid -> Dropout -> IP + HardTanh -> IP -> Softmax
GEN_A = """
name: "gen_a"
layer { name: "data" type: "Input" top: "data" input_param { shape { dim: 3 dim: 17 dim: 17 } } }
layer { name: "c1" type: "Convolution" bottom: "data" top: "c1" convolution_param { num_output: 64 kernel_size: 5 stride: 2 pad: 1 } }
layer { name: "r1" type: "ReLU" bottom: "c1" top: "c1" }
layer { name: "n1" type: "LRN" bottom: "c1" top: "n1" lrn_param { local_size: 5 alpha: 0.0001 beta: 0.75 k: 1 } }
layer { name: "p1" type: "Pooling" bottom: "n1" top: "p1" pooling_param { pool: MAX kernel_size: 3 stride: 2 pad: 1 } }
layer { name: "c2" type: "Convolution" bottom: "p1" top: "c2" convolution_param { num_output: 32 kernel_size: 3 pad: 1 group: 4 } }
layer { name: "r2" type: "ReLU" bottom: "c2" top: "c2" }
layer { name: "l3" type: "LocallyConnected" bottom: "c2" top: "l3" local_param { num_output: 16 kernel_size: 2 stride: 1 } }
layer { name: "t3" type: "TanH" bottom: "l3" top: "l3" }
layer { name: "p3" type: "Pooling" bottom: "l3" top: "p3" pooling_param { pool: AVE kernel_size: 2 stride: 1 pad: 1 } }
layer { name: "f4" type: "InnerProduct" bottom: "p3" top: "f4" inner_product_param { num_output: 24 } }
layer { name: "s4" type: "Sigmoid" bottom: "f4" top: "f4" }
layer { name: "d4" type: "Dropout" bottom: "f4" top: "f4" dropout_param { dropout_ratio: 0.5 } }
layer { name: "f5" type: "InnerProduct" bottom: "f4" top: "f5" inner_product_param { num_output: 20 } }
layer { name: "h5" type: "HardTanh" bottom: "f5" top: "f5" }
layer { name: "f6" type: "InnerProduct" bottom: "f5" top: "f6" inner_product_param { num_output: 10 } }
layer { name: "prob" type: "Softmax" bottom: "f6" top: "prob" }
"""

# conv -> MAX pool -> LRN (after a pool: the standalone LRN kernel) -> conv(pad) -> AVE pool
# (no pad, ceil overhang) -> IP + TanH -> IP -> Softmax
GEN_B = """
name: "gen_b"
layer { name: "data" type: "Input" top: "data" input_param { shape { dim: 3 dim: 20 dim: 20 } } }
layer { name: "c1" type: "Convolution" bottom: "data" top: "c1" convolution_param { num_output: 32 kernel_size: 3 } }
layer { name: "r1" type: "ReLU" bottom: "c1" top: "c1" }
layer { name: "p1" type: "Pooling" bottom: "c1" top: "p1" pooling_param { pool: MAX kernel_size: 2 stride: 2 } }
layer { name: "n1" type: "LRN" bottom: "p1" top: "n1" lrn_param { local_size: 5 alpha: 0.0001 beta: 0.75 k: 1 } }
layer { name: "c2" type: "Convolution" bottom: "n1" top: "c2" convolution_param { num_output: 48 kernel_size: 3 pad: 1 } }
layer { name: "r2" type: "ReLU" bottom: "c2" top: "c2" }
layer { name: "p2" type: "Pooling" bottom: "c2" top: "p2" pooling_param { pool: AVE kernel_size: 3 stride: 2 } }
layer { name: "f3" type: "InnerProduct" bottom: "p2" top: "f3" inner_product_param { num_output: 40 } }
layer { name: "t3" type: "TanH" bottom: "f3" top: "f3" }
layer { name: "f4" type: "InnerProduct" bottom: "f3" top: "f4" inner_product_param { num_output: 12 } }
layer { name: "prob" type: "Softmax" bottom: "f4" top: "prob" }
"""
# gen_a with an unpadded 3x3/2 MAX pool after the LRN: the shape the lrn+pool kernel fuses
GEN_C = GEN_A.replace('name: "gen_a"', 'name: "gen_c"').replace("kernel_size: 3 stride: 2 pad: 1", "kernel_size: 3 stride: 2")
NETS = {"gen_a": GEN_A, "gen_b": GEN_B, "gen_c": GEN_C}
ROWS = 300          # c1 of gen_a: 300 x 64 output pixels = 150 M tiles of 128 plus a ragged tail
SEED = 0x5EED


def _target(net: OracleNet, i: int) -> float:
    """Target pre-activation std of the parametrised layer at net.layers[i] (the Tonic nets'
    calibration rule, oracle/calibrate.py): 100 before an LRN (its denominator is exercised),
    4 for the logit layer and before a sigmoid, 1 elsewhere."""
    if not any("w_shape" in L for L in net.layers[i + 1:]):
        return 4.0
    for L in net.layers[i + 1:]:
        if L["type"] in ("ReLU", "Dropout"):
            continue
        if L["type"] == "LRN":
            return 100.0
        if L["type"] == "Sigmoid":
            return 4.0
        break
    return 1.0


def gen_net(name: str, grid: str):
    """Seeded inputs U(-1,1) and weights U(-1,1) * sqrt(3 / fan_in), each output channel
    standardised (LSUV, by the fp64 oracle on a 64-row calibration batch) to the target std
    with bias jitter 0.1 * t -- the Tonic nets' recipe, so the logits stay input-sensitive and
    16-bit rounding is not amplified by near-zero rows.  Everything on the path's grid."""
    net = OracleNet(NETS[name])
    shp = tuple(net.input_shape)
    per = int(np.prod(shp))
    h = rng.uniform(SEED ^ 0xCA1, 1, 0, 64 * per, -1.0, 1.0).reshape((64,) + shp)
    W, p = [], 0
    for i, L in enumerate(net.layers):
        if L["type"] in ("Input", "Softmax"):
            continue
        if "w_shape" not in L:
            h = net.apply(L, h)
            continue
        a = np.sqrt(3.0 / L["fan_in"])
        nw, nb = int(np.prod(L["w_shape"])), int(np.prod(L["b_shape"]))
        w = rng.uniform(SEED, 10 + 2 * p, 0, nw, -a, a).reshape(L["w_shape"])
        z = net.apply(L, h, w, np.zeros(L["b_shape"]))
        axes = (0,) if z.ndim == 2 else (0, 2, 3)
        mu, sd = z.mean(axis=axes), z.std(axis=axes)
        sd = np.where(sd > 0, sd, 1.0)
        t = _target(net, i)
        ax = 2 if L["type"] == "LocallyConnected" else 0
        shape = [1] * w.ndim
        shape[ax] = -1
        w = w * (t / sd).reshape(shape)
        jit = rng.uniform(SEED, 11 + 2 * p, 0, nb, -0.1 * t, 0.1 * t).reshape(L["b_shape"])
        bsh = [1] * len(L["b_shape"])
        bsh[0] = -1
        b = (-mu * t / sd).reshape(bsh) + jit
        wg, bg = rng.round_to_grid(w, grid), rng.round_to_grid(b, "fp32")
        W.append({"w": wg, "b": bg})
        h = net.apply(L, h, wg.astype(np.float64), bg.astype(np.float64))
        p += 1
    x = rng.round_to_grid(rng.uniform(SEED, 1, 0, ROWS * per, -1.0, 1.0), grid)
    return net, W, x.reshape((ROWS,) + shp)


def run_lib(text, W, x, prec, mode=dj.DJINN_OUT_LOGITS):
    net = dj.DjinnNet(text, recipes.flat_blob(W), prec, x.shape[0])
    out = net.forward(torch.from_numpy(x).cuda(), mode).cpu().numpy()
    plan = net.plan()
    net.close()
    return out, plan


# Measured on B200 (round 2): bf16 activation storage through an LRN at calibrated scale (std 100
# before it) misses the 2e-2 logit bound on the LRN nets -- relL2 max 3.5e-2 (gen_a), 4.4e-2
# (gen_c) -- as it misses top-1 on IMC (tests/parity.py BF16_MISSES); fp16 passes on the same
# inputs.  Strict xfails: a pass would flag a change.
_BF16_LRN = "bf16 storage error through LRN exceeds 2e-2 (relL2 3.5e-2 / 4.4e-2 measured; fp16 passes)"


def _gen_params():
    out = []
    for name in NETS:
        for prec in ("fp32", "bf16", "fp16"):
            marks = [pytest.mark.xfail(strict=True, reason=_BF16_LRN)] if prec == "bf16" and name != "gen_b" else []
            out.append(pytest.param(name, prec, marks=marks, id=f"{name}-{prec}"))
    return out


@pytest.mark.parametrize("name,prec", _gen_params())
def test_generic_net_matches_oracle(name, prec):
    net, W, x = gen_net(name, prec)
    lg_ref, pr_ref = net.forward(x, W)
    lg, plan = run_lib(NETS[name], W, x, prec)
    print(plan)
    if prec == "fp32":
        pr, _ = run_lib(NETS[name], W, x, prec, dj.DJINN_OUT_PROB)
        r = compare_fp32(pr, pr_ref, lg, lg_ref)
        print(name, prec, r)
        assert r["prob_max_abs"] <= FP32_PROB_TOL, r
    else:
        r = compare_16bit(lg, lg_ref)
        print(name, prec, r)
        assert r["rel_max"] <= REL_LOGIT_TOL, r
        assert r["elem_max"] <= ELEM_TOL, r
        assert r["top1_decidable"] >= 0.99, r


_CHILD = r"""
import sys, numpy as np, torch
sys.path.insert(0, sys.argv[1]); sys.path.insert(0, sys.argv[1] + "/tests")
import test_layers_gpu as t
net, W, x = t.gen_net(sys.argv[2], sys.argv[3])
lg, plan = t.run_lib(t.NETS[sys.argv[2]], W, x, sys.argv[3])
print(plan)
np.save(sys.argv[4], lg)
"""


@pytest.mark.parametrize("prec", [pytest.param("bf16", marks=pytest.mark.xfail(strict=True, reason=_BF16_LRN)), "fp16"])
def test_lrn_placements_agree_with_oracle(prec, tmp_path):
    """gen_c's conv1+LRN+pool under every LRN placement (DJINN_LRN_POOL bit 0: LRN in the
    conv epilogue vs the lrn+pool kernel) -- each against the oracle."""
    root = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
    net, W, x = gen_net("gen_c", prec)
    lg_ref, _ = net.forward(x, W)
    plans = []
    for mask in ("0", "1"):
        f = str(tmp_path / f"lg{mask}.npy")
        env = dict(os.environ, DJINN_LRN_POOL=mask)
        out = subprocess.run([sys.executable, "-c", _CHILD, root, "gen_c", prec, f], env=env, check=True,
                             timeout=600, capture_output=True, text=True).stdout
        plans.append(out)
        r = compare_16bit(np.load(f), lg_ref)
        print(mask, r)
        assert r["rel_max"] <= REL_LOGIT_TOL and r["elem_max"] <= ELEM_TOL, r
    assert "lrn-epilogue" in plans[0] and "lrn+pool" in plans[1], plans


@pytest.mark.parametrize("prec", ["fp32", "fp16"])
def test_null_weights_then_arena_copy_reproduces_loaded_net(prec):
    """djinn_load_net(weights=NULL) + a device copy of a loaded net's arena (what the C1 NCCL
    broadcast does on ranks > 0) gives bitwise the loaded net's logits."""
    app = "imc" if prec != "fp32" else "dig"
    n = 5 if app == "imc" else 200
    x = torch.from_numpy(recipes.gen_input_rows(app, 0, n, prec)).cuda()
    a = dj.DjinnNet(dj.net_description(app), blob(app, prec), prec, n)
    b = dj.DjinnNet(dj.net_description(app), None, prec, n)
    ta, tb = parallel.arena_tensor(a), parallel.arena_tensor(b)
    assert ta.numel() == tb.numel()
    tb.copy_(ta)
    torch.cuda.synchronize()
    la = a.forward(x, dj.DJINN_OUT_LOGITS)
    lb = b.forward(x, dj.DJINN_OUT_LOGITS)
    a.close()
    b.close()
    assert torch.equal(la, lb)


def test_unsynced_forward16_then_forward_keep_their_inputs(monkeypatch):
    """host-fed djinn_forward16 followed, without a sync, by host-fed djinn_forward
    on the same net and stream (2 chunks each, so both staging slots are live): each call's
    outputs equal its own device-path reference."""
    app, prec, n = "asr", "fp16", 1024
    monkeypatch.setenv("DJINN_PIPE_CHUNKS", "2")
    xa = recipes.gen_input_rows(app, 0, n, prec)
    xb = recipes.gen_input_rows(app, n, n, prec)
    net = dj.DjinnNet(dj.net_description(app), blob(app, prec), prec, n)
    ra = net.forward(torch.from_numpy(xa).cuda(), dj.DJINN_OUT_LOGITS).cpu()
    rb = net.forward(torch.from_numpy(xb).cuda(), dj.DJINN_OUT_LOGITS).cpu()
    ha16 = torch.from_numpy(xa).half().pin_memory()
    hb = torch.from_numpy(xb).pin_memory()
    s = torch.cuda.Stream()
    outs = []
    for _ in range(3):
        oa = torch.empty(n, net.out_elems).pin_memory()
        ob = torch.empty(n, net.out_elems).pin_memory()
        dj.djinn_forward16(net.handle, ha16, n, oa, dj.DJINN_OUT_LOGITS, s.cuda_stream)
        dj.djinn_forward(net.handle, hb, n, ob, dj.DJINN_OUT_LOGITS, s.cuda_stream)
        outs.append((oa, ob))
    dj.djinn_sync(net.handle, s.cuda_stream)
    net.close()
    for oa, ob in outs:
        assert torch.equal(oa, ra) and torch.equal(ob, rb)


def test_binding_rejects_unsafe_buffers():
    """dtype, contiguity and size are checked before the raw pointers cross the ABI."""
    net = dj.DjinnNet(dj.net_description("pos"), blob("pos", "fp16"), "fp16", 64)
    x = torch.zeros(64, 300, device="cuda")
    out = torch.empty(64, 45, device="cuda")
    cases = [
        (np.zeros((64, 300)), out, dj.DJINN_OUT_PROB),                               # float64 numpy
        (torch.zeros(300, 64, device="cuda").t(), out, dj.DJINN_OUT_PROB),            # non-contiguous
        (torch.zeros(63, 300, device="cuda"), out, dj.DJINN_OUT_PROB),                # too few input rows
        (x, torch.empty(64, 44, device="cuda"), dj.DJINN_OUT_PROB),                   # output too small
        (x, torch.empty(64, device="cuda"), dj.DJINN_OUT_ARGMAX),                     # ARGMAX needs int32
        (x, torch.empty(64, 45, dtype=torch.float16, device="cuda"), dj.DJINN_OUT_PROB),
    ]
    for inp, o, mode in cases:
        with pytest.raises(dj.DjinnError) as e:
            dj.djinn_forward(net.handle, inp, 64, o, mode)
        assert e.value.code == dj.DJINN_E_INVAL
    with pytest.raises(dj.DjinnError):
        dj.djinn_forward16(net.handle, x, 64, out, dj.DJINN_OUT_PROB)                 # fp32 into forward16
    dj.djinn_forward(net.handle, x, 64, out, dj.DJINN_OUT_PROB)                        # the valid call works
    dj.djinn_sync(net.handle)
    net.close()


_SAT_CHILD = r"""
import sys, numpy as np, torch
sys.path.insert(0, sys.argv[1]); sys.path.insert(0, sys.argv[1] + "/tests")
import test_layers_gpu as t
from datagen import recipes
import paper_conf_isca_hauswaldklclmdm15_b200 as dj
net, W, x = t.gen_net("gen_c", "bf16")
W[0]["w"] = W[0]["w"] * 4096.0          # conv1 outputs far beyond the fp16 range (65504)
W[0]["b"] = W[0]["b"] * 4096.0
n = dj.DjinnNet(t.GEN_C, recipes.flat_blob(W), "bf16", x.shape[0])
print(n.plan())
np.save(sys.argv[2], n.forward(torch.from_numpy(x).cuda(), dj.DJINN_OUT_LOGITS).cpu().numpy())
"""


def test_bf16_fp16_intermediate_saturates_instead_of_overflowing(tmp_path):
    """a bf16 net's conv output read only by the lrn+pool kernel is kept in fp16
    ("fp16-out" in the plan); values beyond 65504 must saturate, never become inf / NaN."""
    root = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
    f = str(tmp_path / "lg.npy")
    r = subprocess.run([sys.executable, "-c", _SAT_CHILD, root, f], env=dict(os.environ, DJINN_LRN_POOL="1"),
                       check=True, timeout=600, capture_output=True, text=True)
    assert "fp16-out" in r.stdout, r.stdout
    assert np.isfinite(np.load(f)).all()

"""Whole-net pins of the oracle and of the synthetic-data generator (-m "not gpu")."""
import os

import numpy as np
import pytest
import torch
import torch.nn.functional as F

from datagen import recipes, rng
from oracle import OracleNet
from oracle.calibrate import net_text

GOLD = os.path.join(os.path.dirname(__file__), "golden")
APPS = ["imc", "dig", "face", "asr", "pos", "chk", "ner"]


def _rows(name):
    with open(os.path.join(GOLD, name)) as f:
        return [ln.split() for ln in f if ln.strip() and not ln.startswith("#")]


@pytest.mark.parametrize("app", APPS)
def test_table1_layer_counts(app):
    """PAPER.md Table 1 (L108-118): layer counts.  Counted as Caffe layers excluding
    Input and Softmax; FACE counts DeepFace's C1..F8 (activations folded in) --
    DESIGN.md reading R1."""
    want = {r[0]: int(r[3]) for r in _rows("table1_networks.txt")}[app]
    net = OracleNet(net_text(app))
    excl = ("Input", "Softmax", "ReLU") if app == "face" else ("Input", "Softmax")
    assert net.n_layers(excl) == want


def test_table1_param_count_imc():
    """AlexNet: Table 1 says 60M (L110); the bvlc_alexnet shapes give 60.97M."""
    n = OracleNet(net_text("imc")).n_params()
    assert 60e6 <= n <= 61.5e6


def test_param_counts_of_the_chosen_shapes():
    """Readings R2/R3: our concrete shapes.  Any silent shape change
    (a wrong pool rounding, a wrong LC geometry) moves these counts."""
    want = {"dig": 431080, "face": 102752915, "asr": 38276928, "pos": 103845,
            "chk": 102942, "ner": 117917}
    for app, n in want.items():
        assert OracleNet(net_text(app)).n_params() == n, app


@pytest.mark.parametrize("app", ["imc", "dig", "face"])
def test_table3_input_sizes(app):
    """Table 3 (L155-157): 604 / 307 / 271 KB per query = fp32 input of our shapes."""
    r = {x[0]: x for x in _rows("table3_service.txt")}[app]
    net = OracleNet(net_text(app))
    nbytes = int(r[1]) * int(np.prod(net.input_shape)) * 4
    assert int(r[1]) == net.rows_per_query
    assert abs(nbytes / 1024 - int(r[2])) < 1.0


def test_face_shapes_follow_deepface():
    net = OracleNet(net_text("face"))
    shapes = {L["name"]: L["out_shape"] for L in net.layers}
    assert shapes["C1"] == (32, 142, 142)
    assert shapes["M2"] == (32, 71, 71)
    assert shapes["C3"] == (16, 63, 63)
    assert shapes["L4"] == (16, 55, 55)
    assert shapes["L5"] == (16, 25, 25)
    assert shapes["L6"] == (16, 21, 21)
    assert shapes["F8"] == (83,)


# --------------------------------------------------------------- whole net vs torch
TINY = """
name: "tiny"
layer { name: "data" type: "Input" top: "data" input_param { shape { dim: 3 dim: 17 dim: 17 } } }
layer { name: "c1" type: "Convolution" bottom: "data" top: "c1" convolution_param { num_output: 8 kernel_size: 5 stride: 2 pad: 1 } }
layer { name: "r1" type: "ReLU" bottom: "c1" top: "c1" }
layer { name: "n1" type: "LRN" bottom: "c1" top: "n1" lrn_param { local_size: 5 alpha: 0.0001 beta: 0.75 k: 1 } }
layer { name: "p1" type: "Pooling" bottom: "n1" top: "p1" pooling_param { pool: MAX kernel_size: 3 stride: 2 } }
layer { name: "c2" type: "Convolution" bottom: "p1" top: "c2" convolution_param { num_output: 6 kernel_size: 1 group: 2 } }
layer { name: "l3" type: "LocallyConnected" bottom: "c2" top: "l3" local_param { num_output: 4 kernel_size: 2 stride: 1 } }
layer { name: "t3" type: "TanH" bottom: "l3" top: "l3" }
layer { name: "p3" type: "Pooling" bottom: "l3" top: "p3" pooling_param { pool: AVE kernel_size: 2 stride: 1 pad: 1 } }
layer { name: "f4" type: "InnerProduct" bottom: "p3" top: "f4" inner_product_param { num_output: 7 } }
layer { name: "s4" type: "Sigmoid" bottom: "f4" top: "f4" }
layer { name: "d4" type: "Dropout" bottom: "f4" top: "f4" dropout_param { dropout_ratio: 0.5 } }
layer { name: "f5" type: "InnerProduct" bottom: "f4" top: "f5" inner_product_param { num_output: 5 } }
layer { name: "h5" type: "HardTanh" bottom: "f5" top: "f5" }
layer { name: "f6" type: "InnerProduct" bottom: "f5" top: "f6" inner_product_param { num_output: 3 } }
layer { name: "prob" type: "Softmax" bottom: "f6" top: "prob" }
"""


def _torch_forward(net, x, weights):
    """Library-routine reference: torch fp64 functional ops, LC via unfold."""
    h = torch.from_numpy(x)
    it = iter(weights)
    for L in net.layers[1:]:
        t = L["type"]
        if "w_shape" in L:
            p = next(it)
            w, b = torch.from_numpy(p["w"]), torch.from_numpy(p["b"])
        if t == "Convolution":
            h = F.conv2d(h, w, b, L["stride"], L["pad"], 1, L["group"])
        elif t == "LocallyConnected":
            OH, OW, Co, C, k, _ = w.shape
            cols = F.unfold(h, k, stride=L["stride"])
            h = torch.einsum("nkl,lok->nol", cols, w.reshape(OH * OW, Co, C * k * k))
            h = h.reshape(h.shape[0], Co, OH, OW) + b[None]
        elif t == "InnerProduct":
            h = F.linear(h.reshape(h.shape[0], -1), w, b)
        elif t == "ReLU":
            h = F.relu(h)
        elif t == "Sigmoid":
            h = torch.sigmoid(h)
        elif t == "TanH":
            h = torch.tanh(h)
        elif t == "HardTanh":
            h = F.hardtanh(h)
        elif t == "LRN":
            h = F.local_response_norm(h, L["size"], L["alpha"], L["beta"], L["kk"])
        elif t == "Pooling":
            if L["mode"] == "MAX":
                h = F.max_pool2d(h, L["k"], L["stride"], L["pad"], ceil_mode=True)
            else:
                h = F.avg_pool2d(h, L["k"], L["stride"], L["pad"], ceil_mode=True, count_include_pad=True)
        elif t == "Softmax":
            logits = h
            h = torch.softmax(h, 1)
    return logits.numpy(), h.numpy()


def test_whole_tiny_net_matches_torch_functional():
    net = OracleNet(TINY)
    r = np.random.RandomState(7)
    weights = [{"w": r.randn(*L["w_shape"]) * 0.5, "b": r.randn(*L["b_shape"])} for L in net.param_layers]
    x = 50 * r.randn(4, 3, 17, 17)
    lg, pr = net.forward(x, weights)
    rlg, rpr = _torch_forward(net, x, weights)
    np.testing.assert_allclose(lg, rlg, rtol=1e-11, atol=1e-11)
    np.testing.assert_allclose(pr, rpr, rtol=1e-11, atol=1e-13)


@pytest.mark.parametrize("app", ["dig", "pos", "ner"])
def test_tonic_net_matches_torch_functional(app):
    net = OracleNet(net_text(app))
    W = [{"w": e["w"].astype(np.float64), "b": e["b"].astype(np.float64)}
         for e in recipes.gen_weights(app, "bf16")]
    x = recipes.gen_input_rows(app, 0, 8, "bf16").astype(np.float64)
    lg, pr = net.forward(x, W)
    rlg, rpr = _torch_forward(net, x, W)
    np.testing.assert_allclose(lg, rlg, rtol=1e-10, atol=1e-10)


# --------------------------------------------------------------- generator
def test_generator_is_counter_based_and_shardable():
    a = recipes.gen_input_rows("asr", 0, 100, "fp32")
    b = recipes.gen_input_rows("asr", 37, 20, "fp32")
    np.testing.assert_array_equal(a[37:57], b)
    i1 = recipes.gen_input_rows("face", 0, 3, "bf16")
    i2 = recipes.gen_input_rows("face", 2, 1, "bf16")
    np.testing.assert_array_equal(i1[2:3], i2)


def test_grid_rounding_is_exact_and_idempotent():
    x = np.random.RandomState(3).randn(10000) * 100
    for g in ("bf16", "fp16"):
        r = rng.round_to_grid(x, g)
        np.testing.assert_array_equal(rng.round_to_grid(r, g), r)
    bf = rng.round_to_grid(x, "bf16")
    np.testing.assert_array_equal(bf, torch.from_numpy(x.astype(np.float32)).bfloat16().float().numpy())
    np.testing.assert_array_equal(rng.round_to_grid(x, "fp16"), x.astype(np.float32).astype(np.float16).astype(np.float32))


def test_uniform_and_normal_moments():
    u = rng.uniform(1, 2, 0, 200000)
    assert abs(u.mean() - 0.5) < 0.005 and abs(u.var() - 1 / 12) < 0.002
    z = rng.normal(1, 3, 0, 200000)
    assert abs(z.mean()) < 0.01 and abs(z.std() - 1) < 0.01


@pytest.mark.parametrize("app", ["dig", "pos", "asr"])
def test_calibrated_nets_are_input_sensitive(app):
    """The parity test is non-vacuous: different inputs give different top-1 classes."""
    net = OracleNet(net_text(app))
    W = recipes.gen_weights(app, "fp32")
    x = recipes.gen_input_rows(app, 0, 200, "fp32")
    lg, _ = net.forward(x, W)
    assert len(set(lg.argmax(1).tolist())) >= min(10, lg.shape[1])

"""Pins of the fp64 oracle against things other than itself (-m "not gpu").

Each test ties one oracle function to the paper (golden fixtures with citations),
to a closed form, an invariant, a brute-force or a library routine (PyTorch CPU
fp64 functional ops), chosen so that a dropped term, a wrong sign/index, a
transposed operand or a wrong rounding rule fails at least one test.
"""
import os

import numpy as np
import pytest
import torch
import torch.nn.functional as F

from oracle import ops

GOLD = os.path.join(os.path.dirname(__file__), "golden")
rs = np.random.RandomState(1234)


def t64(a):
    return torch.from_numpy(np.ascontiguousarray(a, dtype=np.float64))


# ------------------------------------------------------------------ convolution
@pytest.mark.parametrize("N,C,H,W,Co,k,s,p,g", [
    (2, 3, 9, 11, 4, 3, 1, 1, 1), (1, 4, 13, 13, 6, 5, 2, 2, 2), (3, 6, 7, 8, 9, 3, 3, 0, 3),
    (1, 3, 23, 23, 5, 11, 4, 0, 1), (2, 8, 6, 6, 8, 1, 1, 0, 4)])
def test_conv_matches_torch(N, C, H, W, Co, k, s, p, g):
    x = rs.randn(N, C, H, W)
    w = rs.randn(Co, C // g, k, k)
    b = rs.randn(Co)
    ref = F.conv2d(t64(x), t64(w), t64(b), stride=s, padding=p, groups=g).numpy()
    y = ops.conv2d(x, w, b, s, p, g)
    assert y.shape == ref.shape
    np.testing.assert_allclose(y, ref, rtol=1e-12, atol=1e-12)


def test_conv_identity_kernel():
    x = rs.randn(2, 5, 6, 7)
    w = np.eye(5).reshape(5, 5, 1, 1)
    np.testing.assert_array_equal(ops.conv2d(x, w, np.zeros(5)), x)


def test_conv_delta_kernel_is_cross_correlation():
    # delta at (ky,kx)=(0,2), pad 1: y[oy,ox] = x[oy-1, ox+1]  (pins orientation + padding)
    x = rs.randn(1, 1, 5, 5)
    w = np.zeros((1, 1, 3, 3))
    w[0, 0, 0, 2] = 1.0
    y = ops.conv2d(x, w, np.zeros(1), 1, 1, 1)
    assert y[0, 0, 1, 2] == x[0, 0, 0, 3]
    assert y[0, 0, 0, 0] == 0.0            # reads the zero pad row
    assert y[0, 0, 4, 4] == 0.0            # reads the zero pad column


def test_conv_groups_are_independent_convs():
    x = rs.randn(2, 6, 7, 7)
    w = rs.randn(4, 3, 3, 3)
    b = rs.randn(4)
    y = ops.conv2d(x, w, b, 1, 1, 2)
    y0 = ops.conv2d(x[:, :3], w[:2], b[:2], 1, 1, 1)
    y1 = ops.conv2d(x[:, 3:], w[2:], b[2:], 1, 1, 1)
    np.testing.assert_array_equal(y, np.concatenate([y0, y1], axis=1))


def test_conv_output_geometry_of_the_tonic_nets():
    assert ops.conv_out(227, 11, 4, 0) == 55      # AlexNet conv1
    assert ops.conv_out(27, 5, 1, 2) == 27        # AlexNet conv2
    assert ops.conv_out(152, 11, 1, 0) == 142     # DeepFace C1
    assert ops.conv_out(55, 7, 2, 0) == 25        # DeepFace L5
    assert ops.conv_out(28, 5, 1, 0) == 24        # LeNet conv1


# ------------------------------------------------------------------ locally connected
def test_local_with_shared_weights_equals_conv():
    x = rs.randn(2, 3, 9, 9)
    wc = rs.randn(4, 3, 3, 3)
    bc = rs.randn(4)
    OH = OW = 4
    wl = np.broadcast_to(wc, (OH, OW, 4, 3, 3, 3)).copy()
    bl = np.broadcast_to(bc[:, None, None], (4, OH, OW)).copy()
    np.testing.assert_allclose(ops.local(x, wl, bl, 2), ops.conv2d(x, wc, bc, 2, 0, 1),
                               rtol=1e-13, atol=1e-13)


def test_local_matches_unfold_einsum():
    x = rs.randn(3, 4, 8, 7)
    k, s = 3, 2
    OH, OW = (8 - k) // s + 1, (7 - k) // s + 1
    w = rs.randn(OH, OW, 5, 4, k, k)
    b = rs.randn(5, OH, OW)
    cols = F.unfold(t64(x), k, stride=s).numpy()            # [N, C*k*k, OH*OW] in (c,ky,kx) order
    wm = w.reshape(OH * OW, 5, 4 * k * k)
    ref = np.einsum("nkl,lok->nol", cols, wm).reshape(3, 5, OH, OW) + b[None]
    np.testing.assert_allclose(ops.local(x, w, b, s), ref, rtol=1e-12, atol=1e-12)


def test_local_location_specificity():
    # weights nonzero at a single location only -> every other location equals its bias
    x = rs.randn(1, 2, 5, 5)
    w = np.zeros((3, 3, 1, 2, 3, 3))
    w[1, 2] = 1.0
    b = np.zeros((1, 3, 3))
    y = ops.local(x, w, b, 1)
    assert y[0, 0, 1, 2] == pytest.approx(x[0, :, 1:4, 2:5].sum())
    assert np.count_nonzero(y) == 1


# ------------------------------------------------------------------ inner product
def test_inner_product_is_matmul():
    x = rs.randn(5, 17)
    w = rs.randn(9, 17)
    b = rs.randn(9)
    np.testing.assert_allclose(ops.inner_product(x, w, b), x @ w.T + b, rtol=1e-12, atol=1e-12)


def test_inner_product_flattens_chw():
    x = rs.randn(2, 3, 2, 2)
    w = np.zeros((1, 12))
    w[0, 1 * 4 + 0 * 2 + 1] = 1.0            # (c=1, h=0, w=1) in Caffe (c,h,w) order
    assert ops.inner_product(x, w, np.zeros(1))[1, 0] == x[1, 1, 0, 1]


# ------------------------------------------------------------------ activations
def test_activations_special_values():
    v = np.array([-2.0, -0.5, 0.0, 0.5, 2.0])
    np.testing.assert_array_equal(ops.activation(v, "ReLU"), [0, 0, 0, 0.5, 2.0])
    np.testing.assert_array_equal(ops.activation(v, "HardTanh"), [-1, -0.5, 0, 0.5, 1])
    assert ops.activation(np.zeros(1), "Sigmoid")[0] == 0.5
    s = ops.activation(v, "Sigmoid")
    np.testing.assert_allclose(s + s[::-1], 1.0, rtol=0, atol=1e-15)     # sigma(-x) = 1 - sigma(x)
    np.testing.assert_allclose(ops.activation(v, "TanH"), np.tanh(v), rtol=0, atol=1e-15)
    np.testing.assert_allclose(s, torch.sigmoid(t64(v)).numpy(), rtol=1e-15)


# ------------------------------------------------------------------ LRN
def _gold(name):
    with open(os.path.join(GOLD, name)) as f:
        return [ln.split() for ln in f if ln.strip() and not ln.startswith("#")]


def test_lrn_constant_input_closed_form():
    g = {k: float(v) for k, v in _gold("lrn_constant_input.txt")}
    y = ops.lrn(np.full((1, 8, 2, 2), 100.0))
    assert y[0, 0, 0, 0] == pytest.approx(g["channel0"], abs=1e-4)
    assert y[0, 1, 1, 1] == pytest.approx(g["channel1"], abs=1e-4)
    assert y[0, 4, 0, 1] == pytest.approx(g["interior"], abs=1e-4)
    assert y[0, 7, 0, 0] == pytest.approx(g["channel0"], abs=1e-4)   # symmetric window at the top


def test_lrn_alpha_zero_is_identity():
    x = rs.randn(2, 7, 3, 3)
    np.testing.assert_array_equal(ops.lrn(x, 5, 0.0, 0.75, 1.0), x)


@pytest.mark.parametrize("C", [3, 5, 16, 96])
def test_lrn_matches_torch(C):
    x = 60.0 * rs.randn(2, C, 4, 5)
    ref = F.local_response_norm(t64(x), 5, alpha=1e-4, beta=0.75, k=1.0).numpy()
    np.testing.assert_allclose(ops.lrn(x), ref, rtol=1e-12, atol=1e-12)


# ------------------------------------------------------------------ pooling
@pytest.mark.parametrize("H,W,k,s,p", [(55, 55, 3, 2, 0), (13, 13, 3, 2, 0), (142, 142, 3, 2, 0),
                                        (24, 24, 2, 2, 0), (7, 8, 3, 2, 1), (10, 9, 3, 3, 1),
                                        (6, 6, 2, 2, 1)])
def test_pool_matches_torch_ceil_mode(H, W, k, s, p):
    x = rs.randn(2, 3, H, W)
    ref_max = F.max_pool2d(t64(x), k, s, p, ceil_mode=True).numpy()
    ref_ave = F.avg_pool2d(t64(x), k, s, p, ceil_mode=True, count_include_pad=True).numpy()
    np.testing.assert_array_equal(ops.pool(x, "MAX", k, s, p), ref_max)
    np.testing.assert_allclose(ops.pool(x, "AVE", k, s, p), ref_ave, rtol=1e-13, atol=1e-14)


def test_pool_geometry_pins():
    assert ops.pool_out(142, 3, 2, 0) == 71      # DeepFace M2: ceil (floor would give 70)
    assert ops.pool_out(55, 3, 2, 0) == 27       # AlexNet pool1
    assert ops.pool_out(13, 3, 2, 0) == 6        # AlexNet pool5
    assert ops.pool_out(24, 2, 2, 0) == 12       # LeNet pool1


def test_max_pool_is_window_max_and_clips_last_window():
    x = np.arange(142 * 142, dtype=np.float64).reshape(1, 1, 142, 142)   # ramp
    y = ops.pool(x, "MAX", 3, 2, 0)
    assert y.shape == (1, 1, 71, 71)
    assert y[0, 0, 70, 70] == x[0, 0, 141, 141]          # last window = rows/cols 140..141
    assert y[0, 0, 3, 5] == x[0, 0, 8, 12]               # window rows 6..8, cols 10..12


def test_ave_pool_constant_interior():
    y = ops.pool(np.full((1, 2, 9, 9), 3.0), "AVE", 3, 2, 1)
    assert y[0, 1, 2, 2] == 3.0
    assert y[0, 0, 0, 0] == pytest.approx(3.0 * 4 / 9)    # pad counted in the divisor


# ------------------------------------------------------------------ softmax / argmax
def test_softmax_textbook_and_invariants():
    g = [float(v) for v in _gold("softmax_123.txt")[0]]
    np.testing.assert_allclose(ops.softmax(np.array([[1.0, 2.0, 3.0]]))[0], g, atol=5e-8)
    z = 10 * rs.randn(6, 1000)
    p = ops.softmax(z)
    np.testing.assert_allclose(p.sum(1), 1.0, atol=1e-12)
    np.testing.assert_allclose(ops.softmax(z + 123.0), p, rtol=1e-12, atol=1e-15)
    np.testing.assert_allclose(ops.softmax(np.full((1, 8), 7.0)), 1 / 8)
    np.testing.assert_allclose(p, torch.softmax(t64(z), 1).numpy(), rtol=1e-12, atol=1e-16)


def test_argmax_ties_lowest_index():
    z = np.array([[0.0, 3.0, 1.0, 3.0], [5.0, 5.0, 5.0, 5.0]])
    np.testing.assert_array_equal(ops.argmax(z), [1, 0])


# ---------------------------------------------------------------- SENNA window lookup (f3)
def test_embedding_hand_example():
    """Window 2 over tables A (3 x 2) and B (2 x 1), word-major ids (a0, b0, a1, b1):
    the row is A[a0] ++ B[b0] ++ A[a1] ++ B[b1] (SENNA window concatenation)."""
    A = np.array([[1., 2.], [3., 4.], [5., 6.]])
    B = np.array([[7.], [8.]])
    tables = np.concatenate([A.ravel(), B.ravel()])
    ids = np.array([[2, 1, 0, 0], [1, 0, 1, 1]], dtype=np.float32)
    y = ops.embedding(ids, tables, 2, [3, 2], [2, 1])
    np.testing.assert_array_equal(y, [[5, 6, 8, 1, 2, 7], [3, 4, 7, 3, 4, 8]])


def test_embedding_equals_one_hot_matmul():
    """Lookup = one-hot(ids) @ table for every (word, table) block."""
    r = np.random.default_rng(5)
    vocab, dims, window = [7, 3, 4], [4, 2, 3], 3
    tabs = [r.standard_normal((v, d)) for v, d in zip(vocab, dims)]
    ids = np.stack([r.integers(0, v, size=(11, window)) for v in vocab], axis=2).reshape(11, -1)
    y = ops.embedding(ids, np.concatenate([t.ravel() for t in tabs]), window, vocab, dims)
    blocks = []
    for w in range(window):
        for t, v in enumerate(vocab):
            onehot = np.eye(v)[ids[:, w * len(vocab) + t]]
            blocks.append(onehot @ tabs[t])
    np.testing.assert_allclose(y, np.concatenate(blocks, axis=1), rtol=0, atol=0)


def test_embedding_invalid_index_selects_zero_vector():
    tables = np.arange(1., 7.)                    # one table 3 x 2
    ids = np.array([[-1.], [3.], [1.5], [2.]])
    y = ops.embedding(ids, tables, 1, [3], [2])
    np.testing.assert_array_equal(y, [[0, 0], [0, 0], [0, 0], [5, 6]])


@pytest.mark.parametrize("app", ["pos_ids", "chk_ids", "ner_ids"])
def test_id_nets_equal_base_net_on_gathered_windows(app):
    """An *_ids net = lookup followed by exactly the base app's MLP; its input is 4 B per
    feature index instead of 4 B per window-vector element."""
    from datagen import recipes
    from oracle import OracleNet
    from oracle.calibrate import net_text
    W = recipes.gen_weights(app, "bf16")
    x = recipes.gen_input_rows(app, 0, 20, "bf16")
    net = OracleNet(net_text(app))
    base = OracleNet(net_text(app[:3]))
    assert net.n_layers() == base.n_layers() + 1
    assert base.input_shape[0] / net.input_shape[0] >= 12      # >= 12x fewer input bytes per row
    lg, _ = net.forward(x, W)
    emb = ops.embedding(x, W[0]["w"], net.layers[1]["window"], net.layers[1]["vocab"], net.layers[1]["dims"])
    lg2, _ = base.forward(emb, W[1:])
    np.testing.assert_array_equal(lg, lg2)

"""CPU emulation of an FP8 (e4m3, tcgen05 kind::f8f6f4) forward pass, to decide whether SURVEY.md
8(f) f4's FP8 path could meet the north_star contract (relL2 <= 2e-2 and top-1 >= 99.9 % on the
logits) before writing its kernels.

Rounding points (the cheapest FP8 scheme a tensor-core path would use): every weighted layer's
weights in e4m3 with a per-output-channel scale (amax / 448), every stored activation (the same
points the 16-bit path stores: after each activation / pooling / LRN) in e4m3 with one per-tensor
scale per batch (amax / 448, computed on the batch itself -- the most favourable dynamic scaling);
accumulation and the logits exact (fp64 here, fp32 on the GPU).  Everything else is the fp64
oracle's layer functions.

usage: python tools/emulate_fp8.py APP [ROWS]      (APP: asr / dig / pos / chk / ner / imc / face)
"""
import os
import sys

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
sys.path.insert(0, os.path.join(ROOT, "tests"))

from datagen import recipes  # noqa: E402
from oracle import OracleNet  # noqa: E402
from oracle.calibrate import net_text  # noqa: E402
from parity import compare_16bit, oracle_rows  # noqa: E402

E4M3_MAX = 448.0


def round_e4m3(v):
    """Round to the e4m3 grid (3 mantissa bits, min normal exponent -6, subnormal step 2^-9),
    half to even, saturating at +-448."""
    v = np.asarray(v, np.float64)
    a = np.abs(v)
    e = np.floor(np.log2(np.where(a > 0, a, 1.0)))
    q = np.exp2(np.maximum(e, -6.0) - 3.0)
    r = np.round(v / q) * q
    return np.clip(r, -E4M3_MAX, E4M3_MAX)


def quant_tensor(h):
    s = np.abs(h).max() / E4M3_MAX
    return h if s == 0 else round_e4m3(h / s) * s


def quant_weights(w):
    w = np.asarray(w, np.float64)
    ax = tuple(range(1, w.ndim))
    s = np.abs(w).max(axis=ax, keepdims=True) / E4M3_MAX
    s = np.where(s > 0, s, 1.0)
    return round_e4m3(w / s) * s


def emulate(app, x):
    net = OracleNet(net_text(app))
    W = recipes.gen_weights(app, "fp32")
    it = iter(W)
    h = np.asarray(x, np.float64).reshape((x.shape[0],) + tuple(net.input_shape))
    h = quant_tensor(h)  # the first layer's A operand
    layers = net.layers[1:]
    for i, L in enumerate(layers):
        t = L["type"]
        if t == "Softmax":
            return h.reshape(h.shape[0], -1)
        if "w_shape" in L:
            p = next(it)
            h = net.apply(L, h, quant_weights(p["w"]), p["b"].astype(np.float64))
            nxt = layers[i + 1]["type"] if i + 1 < len(layers) else ""
            if nxt in ("ReLU", "Sigmoid", "TanH", "HardTanh", "Softmax"):
                continue  # stored after the activation; logits stay wide
            h = quant_tensor(h)
        elif t in ("ReLU", "TanH", "HardTanh", "Pooling", "LRN"):
            h = quant_tensor(net.apply(L, h))
        elif t == "Sigmoid":  # centered storage, as the 16-bit path
            h = quant_tensor(net.apply(L, h) - 0.5) + 0.5
        else:
            h = net.apply(L, h)
    return h.reshape(h.shape[0], -1)


def main():
    app = sys.argv[1]
    rows = int(sys.argv[2]) if len(sys.argv) > 2 else {"asr": 300, "imc": 32, "face": 32}.get(app, 1000)
    x = recipes.gen_input_rows(app, 0, rows, "fp32")
    ref, _ = oracle_rows(app, x, "fp32")
    lg = emulate(app, x)
    r = compare_16bit(lg, ref)
    print(app, "e4m3 emulation", {k: (round(v, 5) if isinstance(v, float) else v) for k, v in r.items()})


if __name__ == "__main__":
    main()

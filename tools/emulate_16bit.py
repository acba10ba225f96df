"""CPU emulation of the 16-bit path's rounding points, to show where its logit error comes from
(DESIGN.md sec 2): the oracle's fp64 layer functions, with every tensor the GPU stores in 16 bits
rounded to that grid (weights and inputs are already on it).  Stored tensors: the output of each
weighted layer after its activation (ASR's sigmoid layers store sigma - 1/2, the consumer's bias
absorbs the 1/2), of each pooling and LRN layer; logits stay fp32.

usage: python tools/emulate_16bit.py APP GRID [ROWS]      (APP: asr / dig / pos / chk / ner)
Prints the emulation's relL2 / top-1 statistics against the unrounded oracle -- the same numbers
tests/parity.py computes for the GPU (e.g. ASR bf16: relL2 max 7.9e-3, top-1 99.69 % of
decidable rows on 1000 frames; GPU: 8.4e-3 / 99.81 % on 8192).
"""
import os
import sys

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
sys.path.insert(0, os.path.join(ROOT, "tests"))

from datagen import recipes, rng  # noqa: E402
from oracle import OracleNet  # noqa: E402
from oracle.calibrate import net_text  # noqa: E402
from parity import compare_16bit, oracle_rows  # noqa: E402


def emulate(app, grid, x):
    net = OracleNet(net_text(app))
    W = recipes.gen_weights(app, grid)
    it = iter(W)
    h = np.asarray(x, np.float64).reshape((x.shape[0],) + tuple(net.input_shape))
    layers = net.layers[1:]
    logits = None
    for i, L in enumerate(layers):
        t = L["type"]
        if t == "Softmax":
            logits = h.reshape(h.shape[0], -1)
            break
        if "w_shape" in L:
            p = next(it)
            h = net.apply(L, h, p["w"].astype(np.float64), p["b"].astype(np.float64))
            nxt = layers[i + 1]["type"] if i + 1 < len(layers) else ""
            if nxt in ("ReLU", "Sigmoid", "TanH", "HardTanh"):
                continue  # stored after the activation
            if nxt == "Softmax":
                continue  # fp32 logits
            h = rng.round_to_grid(h, grid).astype(np.float64)
        elif t in ("ReLU", "TanH", "HardTanh"):
            h = rng.round_to_grid(net.apply(L, h), grid).astype(np.float64)
        elif t == "Sigmoid":  # centered storage: sigma - 1/2 rounded, + 1/2 exact
            s = net.apply(L, h)
            h = rng.round_to_grid(s - 0.5, grid).astype(np.float64) + 0.5
        elif t in ("Pooling", "LRN"):
            h = rng.round_to_grid(net.apply(L, h), grid).astype(np.float64)
        else:
            h = net.apply(L, h)
    return logits


def main():
    app, grid = sys.argv[1], sys.argv[2]
    n = int(sys.argv[3]) if len(sys.argv) > 3 else 1000
    x = recipes.gen_input_rows(app, 0, n, grid)
    lg_ref, _ = oracle_rows(app, x, grid)
    print(app, grid, "emulated rounding vs oracle:", compare_16bit(emulate(app, grid, x), lg_ref))


if __name__ == "__main__":
    main()

"""ORACLE -- test infrastructure only.  Writes datagen/calib/<net>.json.

LSUV-style data-dependent calibration of the synthetic weights (SURVEY.md sec 8(c)
"Proposal: LSUV-style data-dependent init"), computed with the fp64 oracle ONLY:
for each parametrised layer in net order, the raw draws are applied to the
calibrated activations of a fixed calibration batch; each output channel c of the
pre-activation gets   scale_c = t / sigma_c,  shift_c = -mu_c * t / sigma_c,
jitter = 0.1 * t, so that the pre-activation is standardised to std t.
Target std t: 100 for layers feeding an LRN (so that LRN's denominator is genuinely
exercised), 4 for the final (logit) layer and for sigmoid layers (ASR "gain 4"),
1 elsewhere.  Trained weights are unavailable (PAPER.md L94-104 models are OUT of
scope), so this keeps the outputs input-sensitive and the parity test non-vacuous.

Usage:  python -m oracle.calibrate [net ...]
"""
from __future__ import annotations

import json
import os
import sys
import time

import numpy as np

from datagen import recipes
from .net import OracleNet

NETS_DIR = os.path.join(os.path.dirname(os.path.dirname(os.path.abspath(__file__))),
                        "paper_conf_isca_hauswaldklclmdm15_b200", "nets")
CALIB_ROWS = {"imc": 32, "face": 32, "dig": 64, "asr": 512, "pos": 512, "chk": 512, "ner": 512}


def net_text(app: str) -> str:
    with open(os.path.join(NETS_DIR, f"{app}.prototxt")) as f:
        return f.read()


def _target(net: OracleNet, i: int) -> float:
    """Target pre-activation std for the parametrised layer at index i of net.layers."""
    rest = net.layers[i + 1:]
    if not any("w_shape" in L for L in rest):
        return 4.0
    for L in rest:
        if L["type"] in ("ReLU", "Dropout"):
            continue
        if L["type"] == "Sigmoid":
            return 4.0
        if L["type"] == "LRN":
            return 100.0
        break
    return 1.0


def calibrate(app: str) -> dict:
    net = OracleNet(net_text(app))
    h = recipes.calib_input_rows(app, CALIB_ROWS[app])
    entries = []
    p = 0
    for i, L in enumerate(net.layers):
        if L["type"] in ("Input", "Softmax"):
            continue
        if "w_shape" not in L:
            h = net.apply(L, h)
            continue
        w = recipes.raw_weight(app, p, L["w_shape"], L["fan_in"])
        z = net.apply(L, h, w, np.zeros(L["b_shape"]))
        axes = (0,) if z.ndim == 2 else (0, 2, 3)
        mu, sd = z.mean(axis=axes), z.std(axis=axes)
        sd = np.where(sd > 0, sd, 1.0)
        t = _target(net, i)
        e = {"layer": L["name"], "type": L["type"], "w_shape": list(L["w_shape"]),
             "b_shape": list(L["b_shape"]), "fan_in": int(L["fan_in"]), "target_std": t,
             "scale": [float(v) for v in t / sd], "shift": [float(v) for v in -mu * t / sd],
             "jitter": 0.1 * t}
        entries.append(e)
        wf, bf = recipes.scale_weights(app, e, p)
        h = net.apply(L, h, wf, bf)
        p += 1
    return {"net": app, "calib_rows": CALIB_ROWS[app],
            "generator": "oracle/calibrate.py (fp64 oracle only)", "params": entries}


def main(argv):
    apps = argv or ["dig", "pos", "chk", "ner", "asr", "face", "imc"]
    for app in apps:
        t0 = time.time()
        c = calibrate(app)
        with open(os.path.join(recipes.CALIB_DIR, f"{app}.json"), "w") as f:
            json.dump(c, f)
        print(f"{app}: {len(c['params'])} layers calibrated in {time.time() - t0:.1f}s")


if __name__ == "__main__":
    main(sys.argv[1:])

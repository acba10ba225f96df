"""Seeded synthetic inputs and weights of the Tonic networks' shapes.

The recipe (SURVEY.md sec 8(c) "Synthetic data that makes parity meaningful",
restated in DESIGN.md sec 3):

* IMC / FACE images: per-image channel offsets + a random-direction gradient +
  4 Gaussian blobs + uniform noise, clipped to +-128 (the "mean-subtracted 0-255"
  range of Caffe image nets).  Shapes 3x227x227 / 3x152x152 (Table 3 input sizes
  604 KB / 271 KB = 4-byte floats).
* DIG: pixels k/256, k ~ U{0..255}, 1x28x28; a query is 100 images (L156).
* ASR: N(0,1) per feature (CMVN-like), 440-dim rows; a query is 548 rows (L158).
* POS/CHK/NER: U(-1,1) window vectors (300 / 300 / 375); a query is 28 rows (L159-161).
* POS/CHK/NER with the on-GPU SENNA lookup (``*_ids``): per window word
  the table indices, word index floor(V * u^3) (skewed toward frequent words, Zipf-like),
  the other features uniform; tables U(-1,1) (the same marginal as the window vectors
  above), followed by exactly the base app's MLP weights.
* Weights: raw_W ~ U(-1,1) * sqrt(3 / fan_in), then multiplied per output channel
  by a stored calibration scale; bias = stored per-channel shift + jitter * U(-1,1).
  The calibration vectors are written by ``oracle/calibrate.py`` (which calls only
  ``oracle/``) into ``datagen/calib/<net>.json`` -- this module only reads them.

Nothing here evaluates a layer: the only arithmetic is drawing, scaling by a stored
vector, clipping the synthetic image and rounding to the storage grid.
"""
from __future__ import annotations

import json
import os
from typing import Dict, List, Tuple

import numpy as np

from . import rng

CALIB_DIR = os.path.join(os.path.dirname(os.path.abspath(__file__)), "calib")

# Per-app input geometry (C, H, W) or (K,) and rows per query (Table 3).
INPUT_SHAPE = {
    "imc": (3, 227, 227), "dig": (1, 28, 28), "face": (3, 152, 152), "asr": (440,),
    "pos": (300,), "chk": (300,), "ner": (375,),
    "pos_ids": (15,), "chk_ids": (15,), "ner_ids": (30,),
}
ROWS_PER_QUERY = {"imc": 1, "dig": 100, "face": 1, "asr": 548, "pos": 28, "chk": 28, "ner": 28,
                  "pos_ids": 28, "chk_ids": 28, "ner_ids": 28}
# token-id apps: (base app whose MLP follows, window, table vocabularies) -- the tables' dims
# live in the net description; the generator only needs the index ranges
ID_APPS = {"pos_ids": ("pos", 5, (130000, 5, 455)), "chk_ids": ("chk", 5, (130000, 5, 45)),
           "ner_ids": ("ner", 5, (130000, 5, 2, 2, 2, 2))}
ID_TABLE_DIMS = {"pos_ids": (50, 5, 5), "chk_ids": (50, 5, 5), "ner_ids": (50, 5, 5, 5, 5, 5)}
_TID_TABLES = 90

_TID_NOISE, _TID_IMG = 1, 2
CALIB_SEED_XOR = 0xCA11B


def _structured_images(seed: int, start: int, n: int, c: int, h: int, w: int) -> np.ndarray:
    P = 4 + 4 * (3 + c)          # per-image parameter draws
    per = c * h * w
    out = np.empty((n, c, h, w), dtype=np.float64)
    yy, xx = np.meshgrid(np.arange(h, dtype=np.float64), np.arange(w, dtype=np.float64), indexing="ij")
    for i in range(n):
        g = start + i
        p = rng.uniform(seed, _TID_IMG, g * P, P)
        theta = 2.0 * np.pi * p[0]
        amp = 20.0 + 40.0 * p[1]
        off = -30.0 + 60.0 * rng.uniform(seed, _TID_IMG + 1, g * c, c)
        grad = amp * ((xx - w / 2) * np.cos(theta) + (yy - h / 2) * np.sin(theta)) / (w / 2)
        img = np.empty((c, h, w))
        for ch in range(c):
            img[ch] = off[ch] + grad
        for b in range(4):
            q = p[4 + b * (3 + c): 4 + (b + 1) * (3 + c)]
            cy, cx = q[0] * h, q[1] * w
            sig = w / 20.0 + (w / 5.0 - w / 20.0) * q[2]
            blob = np.exp(-((yy - cy) ** 2 + (xx - cx) ** 2) / (2.0 * sig * sig))
            for ch in range(c):
                img[ch] += (-80.0 + 160.0 * q[3 + ch]) * blob
        noise = rng.uniform(seed, _TID_NOISE, g * per, per, -20.0, 20.0).reshape(c, h, w)
        out[i] = np.clip(img + noise, -128.0, 128.0)
    return out


def gen_input_rows(app: str, start_row: int, n_rows: int, grid: str = "fp32",
                   seed: int | None = None) -> np.ndarray:
    """Rows [start_row, start_row + n_rows) of the app's synthetic query stream, float32,
    shaped (n_rows, *INPUT_SHAPE[app]) in Caffe NCHW row order, rounded onto ``grid``."""
    seed = rng.app_seed(app) if seed is None else seed
    shp = INPUT_SHAPE[app]
    per = int(np.prod(shp))
    if app in ("imc", "face"):
        x = _structured_images(seed, start_row, n_rows, *shp)
    elif app == "dig":
        k = np.floor(rng.uniform(seed, _TID_NOISE, start_row * per, n_rows * per) * 256.0)
        x = (k / 256.0).reshape((n_rows,) + shp)
    elif app == "asr":
        x = rng.normal(seed, _TID_NOISE, start_row * per, n_rows * per).reshape((n_rows,) + shp)
    elif app in ("pos", "chk", "ner"):
        x = rng.uniform(seed, _TID_NOISE, start_row * per, n_rows * per, -1.0, 1.0).reshape((n_rows,) + shp)
    elif app in ID_APPS:
        _, window, vocab = ID_APPS[app]
        u = rng.uniform(seed, _TID_NOISE, start_row * per, n_rows * per).reshape(n_rows, window, len(vocab))
        u[:, :, 0] = u[:, :, 0] ** 3
        x = np.floor(u * np.asarray(vocab, dtype=np.float64)).reshape(n_rows, per)
        return x.astype(np.float32)      # indices: exact integers, no grid rounding
    else:
        raise ValueError(app)
    return rng.round_to_grid(x, grid)


def calib_input_rows(app: str, n_rows: int) -> np.ndarray:
    """The fixed calibration batch (a seed disjoint from the evaluation stream), fp64."""
    return gen_input_rows(app, 0, n_rows, "fp32", seed=rng.app_seed(app) ^ CALIB_SEED_XOR).astype(np.float64)


# --------------------------------------------------------------------------- weights

def raw_weight(app: str, p: int, w_shape: Tuple[int, ...], fan_in: int) -> np.ndarray:
    """Unscaled weights of the p-th parametrised layer: U(-1,1)*sqrt(3/fan_in), fp64."""
    n = int(np.prod(w_shape))
    a = np.sqrt(3.0 / fan_in)
    return rng.uniform(rng.app_seed(app), 100 + 2 * p, 0, n, -a, a).reshape(w_shape)


def bias_jitter(app: str, p: int, b_shape: Tuple[int, ...]) -> np.ndarray:
    n = int(np.prod(b_shape))
    return rng.uniform(rng.app_seed(app), 101 + 2 * p, 0, n, -1.0, 1.0).reshape(b_shape)


def out_channel_axis(layer_type: str) -> int:
    """Axis of the output channel in the canonical weight blob of each layer type
    (Convolution [Co,Ci/g,kh,kw]; InnerProduct [No,K];
    LocallyConnected [OH,OW,Co,Ci,kh,kw])."""
    return 2 if layer_type == "LocallyConnected" else 0


def load_calib(app: str) -> dict:
    with open(os.path.join(CALIB_DIR, f"{app}.json")) as f:
        return json.load(f)


def scale_weights(app: str, entry: dict, p: int) -> Tuple[np.ndarray, np.ndarray]:
    """Apply a stored calibration entry to the raw draws (fp64, unrounded)."""
    w = raw_weight(app, p, tuple(entry["w_shape"]), entry["fan_in"])
    ax = out_channel_axis(entry["type"])
    sc = np.asarray(entry["scale"], dtype=np.float64)
    shp = [1] * w.ndim
    shp[ax] = -1
    w = w * sc.reshape(shp)
    sh = np.asarray(entry["shift"], dtype=np.float64)
    b_shape = tuple(entry["b_shape"])
    jit = bias_jitter(app, p, b_shape) * float(entry["jitter"])
    bshp = [1] * len(b_shape)
    bshp[0] = -1                      # bias: channel is the leading axis for every type
    b = sh.reshape(bshp) + jit
    return w, b


def gen_weights(app: str, grid: str = "fp32", calib: dict | None = None) -> List[Dict]:
    """All parametrised layers' weights, rounded onto ``grid`` (float32 arrays).

    Returns a list of {"layer", "type", "w", "b"} in net order.  Biases are kept in
    fp32 (the GPU path keeps bias in fp32 for every precision)."""
    if app in ID_APPS:               # lookup tables, then the base app's MLP
        base, _, vocab = ID_APPS[app]
        n = int(sum(v * d for v, d in zip(vocab, ID_TABLE_DIMS[app])))
        tab = rng.uniform(rng.app_seed(app), _TID_TABLES, 0, n, -1.0, 1.0)
        return [{"layer": "emb", "type": "Embedding", "w": rng.round_to_grid(tab, grid),
                 "b": np.zeros(0, np.float32)}] + gen_weights(base, grid)
    calib = load_calib(app) if calib is None else calib
    out = []
    for p, e in enumerate(calib["params"]):
        w, b = scale_weights(app, e, p)
        out.append({"layer": e["layer"], "type": e["type"],
                    "w": rng.round_to_grid(w, grid), "b": rng.round_to_grid(b, "fp32")})
    return out


def flat_blob(weights: List[Dict]) -> np.ndarray:
    """The canonical weight blob: for each parametrised layer in net order, its weights
    then its bias, flattened C-order, little-endian float32 (include/djinn.h)."""
    parts = []
    for e in weights:
        parts.append(np.ascontiguousarray(e["w"], dtype=np.float32).ravel())
        parts.append(np.ascontiguousarray(e["b"], dtype=np.float32).ravel())
    return np.concatenate(parts) if parts else np.zeros(0, np.float32)

"""ORACLE -- test infrastructure only.

Net-description reader and fp64 forward pass.  The description is a subset of
Caffe prototxt (DjiNN runs Caffe's configurable layers; "supporting
more applications simply requires providing DjiNN a pretrained neural network
model").  This parser is independent of the product's C++ parser.

A forward pass is the composition, in file order, of the layers below; Dropout is
the identity at inference (SURVEY.md sec 8(c) reading 12), Softmax is the final layer.
"""
from __future__ import annotations

import re
from typing import Any, Dict, List, Tuple

import numpy as np

from . import ops

_TOK = re.compile(r'"[^"]*"|[{}:]|[^\s{}:"]+')


def parse_prototxt(text: str) -> Dict[str, Any]:
    """Parse into nested dicts; repeated keys become lists."""
    text = "\n".join(line.split("#", 1)[0] for line in text.splitlines())
    toks = _TOK.findall(text)
    pos = 0

    def value(t: str):
        if t.startswith('"'):
            return t[1:-1]
        try:
            return int(t)
        except ValueError:
            try:
                return float(t)
            except ValueError:
                return t

    def block() -> Dict[str, Any]:
        nonlocal pos
        d: Dict[str, Any] = {}
        while pos < len(toks) and toks[pos] != "}":
            key = toks[pos]
            pos += 1
            if toks[pos] == ":":
                pos += 1
                if toks[pos] == "{":
                    pos += 1
                    v = block()
                    pos += 1
                else:
                    v = value(toks[pos])
                    pos += 1
            elif toks[pos] == "{":
                pos += 1
                v = block()
                pos += 1
            else:
                raise ValueError(f"bad token after {key!r}: {toks[pos]!r}")
            d.setdefault(key, []).append(v)
        return d

    return block()


def _one(d: Dict[str, Any], key: str, default=None):
    v = d.get(key)
    if v is None:
        return default
    return v[0]


class OracleNet:
    """fp64 reference network.  ``layers`` is the parsed layer list with shapes."""

    def __init__(self, text: str):
        root = parse_prototxt(text)
        self.name = _one(root, "name")
        self.rows_per_query = _one(root, "rows_per_query", 1)
        self.layers: List[Dict[str, Any]] = []
        shape: Tuple[int, ...] = ()
        for L in root["layer"]:
            t = _one(L, "type")
            e: Dict[str, Any] = {"name": _one(L, "name"), "type": t}
            if t == "Input":
                dims = _one(_one(L, "input_param"), "shape")["dim"]
                shape = tuple(int(d) for d in dims)
                self.input_shape = shape
            elif t == "Convolution":
                p = _one(L, "convolution_param")
                co, k = _one(p, "num_output"), _one(p, "kernel_size")
                s, pad, g = _one(p, "stride", 1), _one(p, "pad", 0), _one(p, "group", 1)
                C, H, W = shape
                e.update(co=co, k=k, stride=s, pad=pad, group=g,
                         w_shape=(co, C // g, k, k), b_shape=(co,), fan_in=(C // g) * k * k)
                shape = (co, ops.conv_out(H, k, s, pad), ops.conv_out(W, k, s, pad))
            elif t == "LocallyConnected":
                p = _one(L, "local_param")
                co, k, s = _one(p, "num_output"), _one(p, "kernel_size"), _one(p, "stride", 1)
                C, H, W = shape
                OH, OW = ops.conv_out(H, k, s, 0), ops.conv_out(W, k, s, 0)
                e.update(co=co, k=k, stride=s, w_shape=(OH, OW, co, C, k, k),
                         b_shape=(co, OH, OW), fan_in=C * k * k)
                shape = (co, OH, OW)
            elif t == "Embedding":
                # SENNA window lookup (ops.embedding): input = window * T indices per row
                p = _one(L, "embedding_param")
                window, vocab, dims = _one(p, "window", 1), list(p["vocab"]), list(p["dim"])
                if len(vocab) != len(dims) or shape != (window * len(vocab),):
                    raise ValueError("Embedding: input must hold window * tables indices")
                e.update(window=window, vocab=vocab, dims=dims,
                         w_shape=(int(sum(v * d for v, d in zip(vocab, dims))),), b_shape=(0,), fan_in=1)
                shape = (window * int(sum(dims)),)
            elif t == "InnerProduct":
                no = _one(_one(L, "inner_product_param"), "num_output")
                K = int(np.prod(shape))
                e.update(no=no, w_shape=(no, K), b_shape=(no,), fan_in=K)
                shape = (no,)
            elif t == "Pooling":
                p = _one(L, "pooling_param")
                k, s, pad = _one(p, "kernel_size"), _one(p, "stride", 1), _one(p, "pad", 0)
                mode = _one(p, "pool", "MAX")
                C, H, W = shape
                e.update(mode=mode, k=k, stride=s, pad=pad)
                shape = (C, ops.pool_out(H, k, s, pad), ops.pool_out(W, k, s, pad))
            elif t == "LRN":
                p = _one(L, "lrn_param")
                e.update(size=_one(p, "local_size", 5), alpha=float(_one(p, "alpha", 1.0)),
                         beta=float(_one(p, "beta", 0.75)), kk=float(_one(p, "k", 1.0)))
            elif t in ("ReLU", "Sigmoid", "TanH", "HardTanh", "Dropout", "Softmax"):
                pass
            else:
                raise ValueError(f"unsupported layer type {t}")
            e["out_shape"] = shape
            self.layers.append(e)
        self.out_dim = int(np.prod(shape))

    # ------------------------------------------------------------------ structure
    @property
    def param_layers(self) -> List[Dict[str, Any]]:
        return [L for L in self.layers if "w_shape" in L]

    def n_params(self) -> int:
        return int(sum(np.prod(L["w_shape"]) + np.prod(L["b_shape"]) for L in self.param_layers))

    def n_layers(self, exclude=("Input", "Softmax")) -> int:
        return sum(1 for L in self.layers if L["type"] not in exclude)

    # ------------------------------------------------------------------ forward
    def apply(self, L: Dict[str, Any], x: np.ndarray, w=None, b=None) -> np.ndarray:
        t = L["type"]
        if t == "Convolution":
            return ops.conv2d(x, w, b, L["stride"], L["pad"], L["group"])
        if t == "LocallyConnected":
            return ops.local(x, w, b, L["stride"])
        if t == "Embedding":
            return ops.embedding(x.reshape(x.shape[0], -1), w, L["window"], L["vocab"], L["dims"])
        if t == "InnerProduct":
            return ops.inner_product(x.reshape(x.shape[0], -1), w, b)
        if t in ("ReLU", "Sigmoid", "TanH", "HardTanh"):
            return ops.activation(x, t)
        if t == "LRN":
            return ops.lrn(x, L["size"], L["alpha"], L["beta"], L["kk"])
        if t == "Pooling":
            return ops.pool(x, L["mode"], L["k"], L["stride"], L["pad"])
        if t == "Dropout":
            return x
        if t == "Softmax":
            return ops.softmax(x.reshape(x.shape[0], -1))
        raise ValueError(t)

    def forward(self, x: np.ndarray, weights: List[Dict[str, Any]]) -> Tuple[np.ndarray, np.ndarray]:
        """x: [rows, *input_shape] (any float dtype, widened to fp64);
        weights: list of {"w","b"} per parametrised layer in net order.
        Returns (logits, probabilities) as fp64 [rows, out_dim]."""
        h = np.asarray(x, dtype=np.float64).reshape((x.shape[0],) + tuple(self.input_shape))
        it = iter(weights)
        logits = None
        for L in self.layers[1:]:
            if L["type"] == "Softmax":
                logits = h.reshape(h.shape[0], -1)
            if "w_shape" in L:
                p = next(it)
                h = self.apply(L, h, np.asarray(p["w"], np.float64), np.asarray(p["b"], np.float64))
            else:
                h = self.apply(L, h)
        if logits is None:
            logits = h.reshape(h.shape[0], -1)
            return logits, ops.softmax(logits)
        return logits, h.reshape(h.shape[0], -1)

"""ORACLE -- test infrastructure only.  ctypes wrappers over oracle_ops.c (fp64, NCHW)."""
from __future__ import annotations

import ctypes
import os
import subprocess

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "oracle_ops.c")
_LIB = os.path.join(_HERE, "liboracle.so")

_D = ctypes.POINTER(ctypes.c_double)
_I = ctypes.c_int
_L = ctypes.c_int64


def build(force: bool = False) -> str:
    """Compile oracle_ops.c with plain gcc (no -ffast-math: no FP reassociation)."""
    if force or not os.path.exists(_LIB) or os.path.getmtime(_LIB) < os.path.getmtime(_SRC):
        subprocess.check_call(["gcc", "-O2", "-fopenmp", "-fPIC", "-shared", "-std=c11",
                               "-o", _LIB, _SRC, "-lm"])
    return _LIB


_lib = None


def lib():
    global _lib
    if _lib is None:
        _lib = ctypes.CDLL(build())
        L = _lib
        L.orc_conv_out.argtypes = [_I, _I, _I, _I]
        L.orc_pool_out.argtypes = [_I, _I, _I, _I]
        L.orc_conv2d.argtypes = [_D, _I, _I, _I, _I, _D, _D, _I, _I, _I, _I, _I, _I, _D]
        L.orc_local.argtypes = [_D, _I, _I, _I, _I, _D, _D, _I, _I, _I, _I, _D]
        L.orc_inner_product.argtypes = [_D, _I, _I, _D, _D, _I, _D]
        for f in ("orc_relu", "orc_sigmoid", "orc_tanh", "orc_hardtanh"):
            getattr(L, f).argtypes = [_D, _L]
        L.orc_lrn.argtypes = [_D, _I, _I, _I, _I, _I, ctypes.c_double, ctypes.c_double,
                              ctypes.c_double, _D]
        L.orc_pool.argtypes = [_D, _I, _I, _I, _I, _I, _I, _I, _I, _I, _D]
        L.orc_softmax.argtypes = [_D, _I, _I, _D]
        L.orc_argmax.argtypes = [_D, _I, _I, ctypes.POINTER(ctypes.c_int32)]
    return _lib


def _p(a: np.ndarray):
    return a.ctypes.data_as(_D)


def _f64(a) -> np.ndarray:
    return np.ascontiguousarray(a, dtype=np.float64)


def conv_out(i, k, s, p):
    return lib().orc_conv_out(i, k, s, p)


def pool_out(i, k, s, p):
    return lib().orc_pool_out(i, k, s, p)


def conv2d(x, w, b, stride=1, pad=0, group=1):
    x, w, b = _f64(x), _f64(w), _f64(b)
    N, C, H, W = x.shape
    Co, _, KH, KW = w.shape
    OH, OW = conv_out(H, KH, stride, pad), conv_out(W, KW, stride, pad)
    y = np.empty((N, Co, OH, OW))
    lib().orc_conv2d(_p(x), N, C, H, W, _p(w), _p(b), Co, KH, KW, stride, pad, group, _p(y))
    return y


def local(x, w, b, stride=1):
    x, w, b = _f64(x), _f64(w), _f64(b)
    N, C, H, W = x.shape
    OH, OW, Co, _, KH, KW = w.shape
    assert (OH, OW) == (conv_out(H, KH, stride, 0), conv_out(W, KW, stride, 0))
    y = np.empty((N, Co, OH, OW))
    lib().orc_local(_p(x), N, C, H, W, _p(w), _p(b), Co, KH, KW, stride, _p(y))
    return y


def inner_product(x, w, b):
    x = _f64(x).reshape(x.shape[0], -1)
    w, b = _f64(w), _f64(b)
    N, K = x.shape
    No = w.shape[0]
    assert w.shape[1] == K
    y = np.empty((N, No))
    lib().orc_inner_product(_p(x), N, K, _p(w), _p(b), No, _p(y))
    return y


def activation(x, kind: str):
    y = _f64(x).copy()
    getattr(lib(), {"ReLU": "orc_relu", "Sigmoid": "orc_sigmoid", "TanH": "orc_tanh",
                    "HardTanh": "orc_hardtanh"}[kind])(_p(y), y.size)
    return y


def lrn(x, size=5, alpha=1e-4, beta=0.75, k=1.0):
    x = _f64(x)
    N, C, H, W = x.shape
    y = np.empty_like(x)
    lib().orc_lrn(_p(x), N, C, H, W, size, alpha, beta, k, _p(y))
    return y


def pool(x, mode: str, kernel: int, stride: int, pad: int = 0):
    x = _f64(x)
    N, C, H, W = x.shape
    OH, OW = pool_out(H, kernel, stride, pad), pool_out(W, kernel, stride, pad)
    y = np.empty((N, C, OH, OW))
    lib().orc_pool(_p(x), N, C, H, W, {"MAX": 0, "AVE": 1}[mode], kernel, kernel, stride, pad, _p(y))
    return y


def softmax(x):
    x = _f64(x)
    N, D = x.shape
    y = np.empty_like(x)
    lib().orc_softmax(_p(x), N, D, _p(y))
    return y


def argmax(x):
    x = _f64(x)
    N, D = x.shape
    out = np.empty(N, dtype=np.int32)
    lib().orc_argmax(_p(x), N, D, out.ctypes.data_as(ctypes.POINTER(ctypes.c_int32)))
    return out


def embedding(ids, tables, window: int, vocab, dims):
    """SENNA window feature vector ("SENNA ... [builds]
    word vectors" for the NLP services; window approach of the cited SENNA work [ext: ref 19]).

    ids    : [rows, window * T] per word w the T feature indices (word, caps, suffix / tag /
             gazetteer ...), word-major: ids[r, w*T + t].
    tables : flat fp64, table t = [vocab[t], dims[t]] C-order, tables back to back.
    Row r of the result is concat over w of concat over t of table_t[ids[r, w*T+t]], i.e.
    out[r, w*D + sum(dims[:t]) + j] with D = sum(dims).  An index that is not an integer in
    [0, vocab[t]) selects the zero vector (reading R17).
    Written as the plain definition: one lookup per (row, word, table)."""
    ids = np.asarray(ids, dtype=np.float64)
    tables = np.asarray(tables, dtype=np.float64).ravel()
    T = len(vocab)
    D = int(sum(dims))
    rows = ids.shape[0]
    out = np.zeros((rows, window * D), dtype=np.float64)
    base = 0
    mats = []
    for t in range(T):
        mats.append(tables[base: base + vocab[t] * dims[t]].reshape(vocab[t], dims[t]))
        base += vocab[t] * dims[t]
    for r in range(rows):
        for w in range(window):
            col = w * D
            for t in range(T):
                v = ids[r, w * T + t]
                if v == np.floor(v) and 0 <= v < vocab[t]:
                    out[r, col: col + dims[t]] = mats[t][int(v)]
                col += dims[t]
    return out

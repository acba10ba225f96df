"""Shared helpers of the GPU parity tests: oracle vs CUDA path on the same seeded inputs.

The oracle consumes exactly the numbers the kernels consume: weights and inputs are
generated on the path's storage grid (datagen.round_to_grid), so the library's own
fp32 -> 16-bit rounding at load is the identity (reading R13).

Tolerances (BASELINE.json north_star; DESIGN.md sec 3 "tolerances"):
  fp32 path : max |p_gpu - p_oracle| <= 1e-4 on the returned probabilities.
  16-bit    : per-row relative logit error ||dz||_2 / ||z||_2 <= 2e-2, and top-1 agreement
              >= 99.9% over decidable rows (oracle top-2 margin >= 1e-2 * rms(z_row)).
"""
from __future__ import annotations

import functools

import numpy as np

from datagen import recipes
from oracle import OracleNet
from oracle.calibrate import net_text

GRID = {"fp32": "fp32", "bf16": "bf16", "fp16": "fp16"}
FP32_PROB_TOL = 1e-4
REL_LOGIT_TOL = 2e-2
TOP1_MIN = 0.999
MARGIN_TAU = 1e-2
# Element-wise bound |dz_j| <= ELEM_TOL * rms(z_row): a per-row relL2 of 2e-2 spread over
# the row makes a typical element error ~2e-2 rms and the maximum over ~1e6-8e7 elements
# (Gaussian tail, ~5.5 sigma) ~0.11 rms; a wrong logit is O(1) rms.
ELEM_TOL = 0.15
# Per-column relative L2 over the evaluated rows (same reasoning, over rows not columns).
COL_REL_TOL = 5e-2
# top-1 agreement is a rate: asserted only over >= TOP1_MIN_ROWS evaluated rows.
TOP1_MIN_ROWS = 1000
# (app -> measured numbers) where the bf16 path misses the contract at full size; the
# full-size test is then an xfail(strict=True) (see tests/test_fullsize_gpu.py).
# Measured on B200 (round 2, every bench-batch row; fp16 on the same inputs: relL2 <= 3.9e-3,
# 0 top-1 misses for every app).  CPU emulation of the bf16 rounding points reproduces the
# misses (tools/emulate_16bit.py; ASR: 7.9e-3, 99.69 %), i.e. they are the format's, not the
# kernels'.
BF16_MISSES: dict = {
    "imc": "bf16 top-1 98.48 % of 989 decidable rows (15 misses), relL2 max 1.95e-2",
    "face": "bf16 top-1 99.70 % of 1003 decidable rows (3 misses), relL2 max 1.35e-2",
    "asr": "bf16 top-1 99.81 % of 7926 decidable rows (15 misses), relL2 max 8.4e-3",
    "dig": "bf16 top-1 99.81 % of 1578 decidable rows (3 misses), relL2 max 1.99e-2",
}


@functools.lru_cache(maxsize=4)
def weights(app: str, grid: str):
    return recipes.gen_weights(app, grid)


@functools.lru_cache(maxsize=8)
def oracle_net(app: str) -> OracleNet:
    return OracleNet(net_text(app))


def blob(app: str, grid: str) -> np.ndarray:
    return recipes.flat_blob(weights(app, grid))


def oracle_rows(app: str, x: np.ndarray, grid: str, chunk: int = 64):
    net = oracle_net(app)
    W = [{"w": e["w"].astype(np.float64), "b": e["b"].astype(np.float64)} for e in weights(app, grid)]
    lg, pr = [], []
    for i in range(0, x.shape[0], chunk):
        a, b = net.forward(x[i:i + chunk], W)
        lg.append(a)
        pr.append(b)
    return np.concatenate(lg), np.concatenate(pr)


def compare_16bit(lg_gpu: np.ndarray, lg_ref: np.ndarray) -> dict:
    """Per-row relative L2 logit error, element-wise error in units of the row's rms logit,
    per-column relative L2 error (over rows: a wrong output column, e.g. in an N-tail tile,
    shows up here at O(1) even when it is 1 of 8000 logits of a row), and top-1 agreement on
    decidable rows (reading R14)."""
    d = lg_gpu.astype(np.float64) - lg_ref
    rel = np.linalg.norm(d, axis=1) / np.maximum(np.linalg.norm(lg_ref, axis=1), 1e-30)
    rms = np.sqrt((lg_ref ** 2).mean(axis=1))
    elem = np.abs(d) / np.maximum(rms, 1e-30)[:, None]
    col = np.linalg.norm(d, axis=0) / np.maximum(np.linalg.norm(lg_ref, axis=0), 1e-30)
    s = np.sort(lg_ref, axis=1)
    margin = (s[:, -1] - s[:, -2]) / np.maximum(rms, 1e-30)
    dec = margin >= MARGIN_TAU
    agree = lg_gpu.argmax(1) == lg_ref.argmax(1)
    return {"rows": int(lg_ref.shape[0]), "rel_max": float(rel.max()), "rel_mean": float(rel.mean()),
            "elem_max": float(elem.max()), "col_rel_max": float(col.max()),
            "top1_raw": float(agree.mean()), "decidable": int(dec.sum()),
            "top1_decidable": float(agree[dec].mean()) if dec.any() else 1.0,
            "top1_misses": int((~agree[dec]).sum())}


def compare_fp32(pr_gpu, pr_ref, lg_gpu, lg_ref) -> dict:
    return {"rows": int(pr_ref.shape[0]), "prob_max_abs": float(np.abs(pr_gpu - pr_ref).max()),
            "logit_max_abs": float(np.abs(lg_gpu - lg_ref).max())}

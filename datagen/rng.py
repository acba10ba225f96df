"""Counter-based random numbers shared by the oracle tests and the product harness.

This module holds NO arithmetic of the method (no layer, no activation, no
normalisation): it only turns (seed, tensor_id, element index) into uniform or
normal deviates, so that any shard of any tensor is generable independently on
any rank (SURVEY.md sec 8(c) "Generation"; sec 8(e) "each rank generates its own
shard").

Generator: splitmix64 finaliser applied to a Weyl sequence.
    key      = mix(seed + G * (tensor_id + 1))
    u64(i)   = mix(key + G * (i + 1))            (mod 2**64)
    U[0,1)   = (u64 >> 11) * 2**-53
with G = 0x9E3779B97F4A7C15.
"""
from __future__ import annotations

import numpy as np

_G = np.uint64(0x9E3779B97F4A7C15)
_M1 = np.uint64(0xBF58476D1CE4E5B9)
_M2 = np.uint64(0x94D049BB133111EB)

# Seeds: 0x15CA2015 ^ app_id.
APP_IDS = {"imc": 1, "dig": 2, "face": 3, "asr": 4, "pos": 5, "chk": 6, "ner": 7,
           "pos_ids": 8, "chk_ids": 9, "ner_ids": 10}


def app_seed(app: str) -> int:
    return 0x15CA2015 ^ APP_IDS[app]


def _mix(z: np.ndarray) -> np.ndarray:
    z = z ^ (z >> np.uint64(30))
    z = z * _M1
    z = z ^ (z >> np.uint64(27))
    z = z * _M2
    return z ^ (z >> np.uint64(31))


def _key(seed: int, tensor_id: int) -> np.uint64:
    with np.errstate(over="ignore"):
        z = np.array([(seed + 0x9E3779B97F4A7C15 * (tensor_id + 1)) % (1 << 64)], dtype=np.uint64)
        return _mix(z)[0]


def u64(seed: int, tensor_id: int, start: int, count: int) -> np.ndarray:
    """Raw 64-bit draws for element indices [start, start+count)."""
    key = _key(seed, tensor_id)
    idx = np.arange(start + 1, start + count + 1, dtype=np.uint64)
    with np.errstate(over="ignore"):
        return _mix(key + _G * idx)


def uniform(seed: int, tensor_id: int, start: int, count: int,
            lo: float = 0.0, hi: float = 1.0) -> np.ndarray:
    """float64 uniform deviates on [lo, hi) for element indices [start, start+count)."""
    u = (u64(seed, tensor_id, start, count) >> np.uint64(11)).astype(np.float64) * (2.0 ** -53)
    return lo + (hi - lo) * u


def normal(seed: int, tensor_id: int, start: int, count: int) -> np.ndarray:
    """float64 N(0,1) deviates (Box-Muller over the draw pairs 2i, 2i+1)."""
    u = uniform(seed, tensor_id, 2 * start, 2 * count).reshape(count, 2)
    u1 = 1.0 - u[:, 0]                      # (0, 1]
    return np.sqrt(-2.0 * np.log(u1)) * np.cos(2.0 * np.pi * u[:, 1])


def round_to_grid(x: np.ndarray, grid: str) -> np.ndarray:
    """Round to the storage grid the GPU path consumes, returned as float32.

    'fp32': plain float32 rounding; 'bf16': round-to-nearest-even to bfloat16;
    'fp16': round-to-nearest-even to IEEE half.  Values produced here are exactly
    representable on the grid, so the library's own fp32 -> 16-bit conversion at
    load is the identity and the oracle sees the very numbers the kernels use
    (SURVEY.md sec 8(c) reading 13).
    """
    f = np.asarray(x, dtype=np.float32)
    if grid == "fp32":
        return f.copy()
    if grid == "fp16":
        return f.astype(np.float16).astype(np.float32)
    if grid == "bf16":
        u = f.view(np.uint32).astype(np.uint64)
        u = (u + np.uint64(0x7FFF) + ((u >> np.uint64(16)) & np.uint64(1))) & np.uint64(0xFFFF0000)
        return u.astype(np.uint32).view(np.float32)
    raise ValueError(f"unknown grid {grid!r}")

"""B200-native DjiNN hot path: Python binding of libdjinn (include/djinn.h).

The binding only marshals arguments: every step of the forward pass runs in the
library's sm_100a kernels.  There is no CPU fallback -- importing works without a
GPU, but loading a net without the built library or without an sm_100 device
raises ``DjinnError``.

PyTorch is used for device memory and streams only (BASELINE.json north_star).
"""
from __future__ import annotations

import ctypes
import os
from typing import Optional

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.environ.get("DJINN_LIB") or os.path.join(_HERE, "libdjinn.so")
NETS_DIR = os.path.join(_HERE, "nets")

DJINN_OK, DJINN_E_INVAL, DJINN_E_PARSE, DJINN_E_SHAPE, DJINN_E_WEIGHTS = 0, -1, -2, -3, -4
DJINN_E_NOMEM, DJINN_E_CUDA, DJINN_E_UNSUPPORTED = -5, -6, -7
DJINN_FP32, DJINN_BF16, DJINN_FP16 = 0, 1, 2
DJINN_MEM_HOST, DJINN_MEM_DEVICE = 0, 1
DJINN_OUT_PROB, DJINN_OUT_ARGMAX, DJINN_OUT_LOGITS = 0, 1, 2
PRECISION = {"fp32": DJINN_FP32, "bf16": DJINN_BF16, "fp16": DJINN_FP16}
EXPORTS = ["djinn_load_net", "djinn_forward", "djinn_forward16", "djinn_sync", "djinn_free", "djinn_net_info",
           "djinn_weight_arena", "djinn_plan_info", "djinn_profile", "djinn_profile_read", "djinn_op_info",
           "djinn_describe", "djinn_batcher_create", "djinn_batcher_submit", "djinn_batcher_wait",
           "djinn_batcher_stats", "djinn_batcher_drive", "djinn_batcher_destroy", "djinn_last_error",
           "djinn_kernel_launches"]
OP_KINDS = ["pack", "gemm", "lrn", "pool", "softmax", "lrn+pool"]


class DjinnError(RuntimeError):
    def __init__(self, code: int, msg: str):
        super().__init__(f"djinn error {code}: {msg}")
        self.code = code


_lib = None


def lib() -> ctypes.CDLL:
    """Load libdjinn.so (built in-tree by build.py).  Fails loudly if it is missing."""
    global _lib
    if _lib is None:
        if not os.path.exists(LIB_PATH):
            raise DjinnError(DJINN_E_CUDA, f"{LIB_PATH} not built; run __graft_entry__.build()")
        L = ctypes.CDLL(LIB_PATH)
        P, I, I64, SZ = ctypes.c_void_p, ctypes.c_int, ctypes.c_int64, ctypes.c_size_t
        L.djinn_load_net.argtypes = [ctypes.c_char_p, SZ, P, SZ, I, I, I, I64, ctypes.POINTER(P)]
        L.djinn_forward.argtypes = [P, P, I64, I, P, I, I, P]
        L.djinn_forward16.argtypes = [P, P, I64, I, P, I, I, P]
        L.djinn_sync.argtypes = [P, P]
        L.djinn_free.argtypes = [P]
        L.djinn_net_info.argtypes = [P] + [ctypes.POINTER(I64)] * 4
        L.djinn_weight_arena.argtypes = [P, ctypes.POINTER(P), ctypes.POINTER(SZ)]
        L.djinn_plan_info.argtypes = [P, ctypes.c_char_p, SZ]
        D = ctypes.c_double
        L.djinn_profile.argtypes = [P, I]
        L.djinn_profile_read.argtypes = [P, ctypes.POINTER(D), ctypes.POINTER(I64), I, I]
        L.djinn_op_info.argtypes = [P, I, ctypes.c_char_p, SZ, ctypes.POINTER(I), ctypes.POINTER(D),
                                    ctypes.POINTER(D), ctypes.POINTER(D)]
        L.djinn_describe.argtypes = [ctypes.c_char_p, SZ, I, I64, ctypes.c_char_p, SZ] + [ctypes.POINTER(I64)] * 4
        L.djinn_batcher_create.argtypes = [P, I64, I64, I, ctypes.POINTER(P)]
        L.djinn_batcher_submit.argtypes = [P, P, I64, P, ctypes.POINTER(I64)]
        L.djinn_batcher_wait.argtypes = [P, I64, I64]
        L.djinn_batcher_stats.argtypes = [P] + [ctypes.POINTER(I64)] * 3 + [ctypes.POINTER(D)] * 2
        L.djinn_batcher_drive.argtypes = [P, P, I64, I64, I, D, ctypes.POINTER(D), ctypes.POINTER(D), ctypes.POINTER(D)]
        L.djinn_batcher_destroy.argtypes = [P]
        L.djinn_last_error.restype = ctypes.c_char_p
        L.djinn_last_error.argtypes = []
        L.djinn_kernel_launches.restype = I64
        L.djinn_kernel_launches.argtypes = []
        for f in EXPORTS[:-2]:
            getattr(L, f).restype = I
        L.djinn_batcher_destroy.restype = I
        _lib = L
    return _lib


def _check(rc: int) -> int:
    if rc < 0:
        raise DjinnError(rc, lib().djinn_last_error().decode())
    return rc


def _ptr_mem(t):
    """(pointer, memory kind) of a torch tensor or numpy array."""
    if isinstance(t, np.ndarray):
        return t.ctypes.data, DJINN_MEM_HOST
    return t.data_ptr(), (DJINN_MEM_DEVICE if t.is_cuda else DJINN_MEM_HOST)


# ----------------------------------------------------------------- C-ABI mirrors
def djinn_load_net(desc: str, weights, precision: int, max_rows: int, device: int = 0) -> int:
    """Mirror of djinn_load_net.  ``weights``: float32 numpy array / torch tensor or None."""
    d = desc.encode()
    h = ctypes.c_void_p()
    if weights is None:
        wp, n, mem = None, 0, DJINN_MEM_HOST
    else:
        if isinstance(weights, np.ndarray):
            weights = np.ascontiguousarray(weights, dtype=np.float32)
        wp, mem = _ptr_mem(weights)
        n = int(weights.size if isinstance(weights, np.ndarray) else weights.numel())
    _check(lib().djinn_load_net(d, len(d), wp, n, mem, device, precision, max_rows, ctypes.byref(h)))
    return h.value


def _dtype_name(t) -> str:
    return str(t.dtype).replace("torch.", "")


def _numel(t) -> int:
    return int(t.size if isinstance(t, np.ndarray) else t.numel())


def _contiguous(t) -> bool:
    return bool(t.flags["C_CONTIGUOUS"]) if isinstance(t, np.ndarray) else bool(t.is_contiguous())


def _validate(net: int, inp, rows: int, out, out_mode: int, in_types) -> None:
    """Argument checks the C ABI cannot make on raw pointers (the library would otherwise
    read or write out of bounds): dtype, contiguity and element counts of both buffers."""
    if rows < 0:
        return                                   # the library reports DJINN_E_INVAL itself
    in_elems, out_elems, _, _ = djinn_net_info(net)
    def bad(msg):
        raise DjinnError(DJINN_E_INVAL, msg)
    if _dtype_name(inp) not in in_types:
        bad(f"input dtype {_dtype_name(inp)}, expected one of {in_types}")
    if not _contiguous(inp):
        bad("input is not C-contiguous")
    if _numel(inp) < rows * in_elems:
        bad(f"input holds {_numel(inp)} elements, {rows} rows need {rows * in_elems}")
    if out_mode == DJINN_OUT_ARGMAX:
        o_types, o_need = ("int32",), rows
    else:
        o_types, o_need = ("float32",), rows * out_elems
    if _dtype_name(out) not in o_types:
        bad(f"output dtype {_dtype_name(out)}, mode {out_mode} needs {o_types[0]}")
    if not _contiguous(out):
        bad("output is not C-contiguous")
    if _numel(out) < o_need:
        bad(f"output holds {_numel(out)} elements, {rows} rows need {o_need}")


def djinn_forward(net: int, inp, rows: int, out, out_mode: int, stream: Optional[int] = None) -> None:
    """Mirror of djinn_forward: ``inp`` float32 rows, ``out`` float32 (int32 for ARGMAX)."""
    _validate(net, inp, rows, out, out_mode, ("float32",))
    ip, imem = _ptr_mem(inp)
    op, omem = _ptr_mem(out)
    _check(lib().djinn_forward(net, ip, rows, imem, op, omem, out_mode, stream))


def djinn_forward16(net: int, inp, rows: int, out, out_mode: int, stream: Optional[int] = None) -> None:
    """Mirror of djinn_forward16: ``inp`` holds the rows in the net's 16-bit type (a torch
    bfloat16 / float16 tensor or a numpy uint16 array of the raw bits)."""
    _validate(net, inp, rows, out, out_mode, ("bfloat16", "float16", "uint16"))
    ip, imem = _ptr_mem(inp)
    op, omem = _ptr_mem(out)
    _check(lib().djinn_forward16(net, ip, rows, imem, op, omem, out_mode, stream))


def djinn_sync(net: int, stream: Optional[int] = None) -> None:
    _check(lib().djinn_sync(net, stream))


def djinn_free(net: int) -> None:
    _check(lib().djinn_free(net))


def djinn_net_info(net: int):
    v = [ctypes.c_int64() for _ in range(4)]
    _check(lib().djinn_net_info(net, *[ctypes.byref(x) for x in v]))
    return tuple(x.value for x in v)


def djinn_weight_arena(net: int):
    p, n = ctypes.c_void_p(), ctypes.c_size_t()
    _check(lib().djinn_weight_arena(net, ctypes.byref(p), ctypes.byref(n)))
    return p.value, n.value


def djinn_plan_info(net: int) -> str:
    n = _check(lib().djinn_plan_info(net, None, 0))
    buf = ctypes.create_string_buffer(n + 1)
    _check(lib().djinn_plan_info(net, buf, n + 1))
    return buf.value.decode()


def djinn_profile(net: int, enable: bool, op: Optional[int] = None) -> None:
    """Per-op device timing on/off; ``op`` = time that plan op only."""
    _check(lib().djinn_profile(net, 0 if not enable else (1 if op is None else 2 + int(op))))


def djinn_profile_read(net: int, reset: bool = True):
    """[(ms_total, launches)] per plan op."""
    n = _check(lib().djinn_profile_read(net, None, None, 0, 0))
    ms = (ctypes.c_double * n)()
    cnt = (ctypes.c_int64 * n)()
    _check(lib().djinn_profile_read(net, ms, cnt, n, 1 if reset else 0))
    return [(ms[i], cnt[i]) for i in range(n)]


def djinn_op_info(net: int, op: int) -> dict:
    name = ctypes.create_string_buffer(128)
    kind = ctypes.c_int()
    f, b, w = ctypes.c_double(), ctypes.c_double(), ctypes.c_double()
    n = _check(lib().djinn_op_info(net, op, name, 128, ctypes.byref(kind), ctypes.byref(f), ctypes.byref(b),
                                   ctypes.byref(w)))
    return {"index": op, "n_ops": n, "name": name.value.decode(), "kind": OP_KINDS[kind.value],
            "flops_per_row": f.value, "bytes_per_row": b.value, "weight_bytes": w.value}


def djinn_describe(desc: str, precision: int, max_rows: int):
    """Host-only planning (no device): (plan text, in_elems, out_elems, n_params, n_layers)."""
    d = desc.encode()
    v = [ctypes.c_int64() for _ in range(4)]
    n = _check(lib().djinn_describe(d, len(d), precision, max_rows, None, 0, *[ctypes.byref(x) for x in v]))
    buf = ctypes.create_string_buffer(n + 1)
    _check(lib().djinn_describe(d, len(d), precision, max_rows, buf, n + 1, None, None, None, None))
    return (buf.value.decode(),) + tuple(x.value for x in v)


def djinn_kernel_launches() -> int:
    return int(lib().djinn_kernel_launches())


# ----------------------------------------------------------------- query batcher
class DjinnBatcher:
    """Mirror of the djinn_batcher_* calls: stacks queries submitted from any thread into
    batches of at most ``max_batch_rows`` rows run by a native worker."""

    def __init__(self, net: "DjinnNet", max_batch_rows: int, max_wait_us: int = 200, out_mode: int = DJINN_OUT_PROB):
        h = ctypes.c_void_p()
        _check(lib().djinn_batcher_create(net.handle, max_batch_rows, max_wait_us, out_mode, ctypes.byref(h)))
        self.handle = h.value
        self.net = net
        self.out_mode = out_mode

    def submit(self, rows: np.ndarray, out: np.ndarray) -> int:
        """Queue one query (float32 C-contiguous host rows); ``out`` (host, float32 rows x
        out_elems, or int32 rows for ARGMAX) must stay alive until wait() returns."""
        if rows.dtype != np.float32 or not rows.flags["C_CONTIGUOUS"]:
            raise DjinnError(DJINN_E_INVAL, "query rows must be C-contiguous float32")
        n = rows.shape[0]
        want = (np.int32, n) if self.out_mode == DJINN_OUT_ARGMAX else (np.float32, n * self.net.out_elems)
        if out.dtype != want[0] or not out.flags["C_CONTIGUOUS"] or out.size < want[1] or \
                rows.size != n * self.net.in_elems:
            raise DjinnError(DJINN_E_INVAL, "query / output buffer shape or dtype")
        t = ctypes.c_int64()
        _check(lib().djinn_batcher_submit(self.handle, rows.ctypes.data, n, out.ctypes.data, ctypes.byref(t)))
        return t.value

    def wait(self, ticket: int, timeout_us: int = -1) -> None:
        _check(lib().djinn_batcher_wait(self.handle, ticket, timeout_us))

    def stats(self) -> dict:
        v = [ctypes.c_int64() for _ in range(3)] + [ctypes.c_double() for _ in range(2)]
        _check(lib().djinn_batcher_stats(self.handle, *[ctypes.byref(x) for x in v]))
        return dict(zip(("batches", "rows", "queries", "p50_us", "p99_us"), (x.value for x in v)))

    def drive(self, queries: np.ndarray, rows_per_query: int, clients: int, seconds: float) -> dict:
        """Native closed-loop load: ``clients`` threads submit-and-wait queries for ``seconds``."""
        q = np.ascontiguousarray(queries, dtype=np.float32)
        n = q.shape[0] // rows_per_query
        qps, p50, p99 = ctypes.c_double(), ctypes.c_double(), ctypes.c_double()
        _check(lib().djinn_batcher_drive(self.handle, q.ctypes.data, n, rows_per_query, clients, seconds,
                                         ctypes.byref(qps), ctypes.byref(p50), ctypes.byref(p99)))
        return {"queries_per_s": qps.value, "p50_us": p50.value, "p99_us": p99.value}

    def close(self) -> None:
        if self.handle:
            _check(lib().djinn_batcher_destroy(self.handle))
            self.handle = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass


# ----------------------------------------------------------------- convenience
def net_description(app: str) -> str:
    with open(os.path.join(NETS_DIR, f"{app}.prototxt")) as f:
        return f.read()


class DjinnNet:
    """A loaded Tonic network (owns the library handle)."""

    def __init__(self, desc: str, weights, precision: str = "bf16", max_rows: int = 1024,
                 device: int = 0):
        self.precision = precision
        self.max_rows = max_rows
        self.device = device
        self.handle = djinn_load_net(desc, weights, PRECISION[precision], max_rows, device)
        self.in_elems, self.out_elems, self.n_params, self.n_layers = djinn_net_info(self.handle)

    def forward(self, x, out_mode: int = DJINN_OUT_PROB, out=None, stream=None, sync: bool = True):
        """x: float32 [rows, ...] torch tensor (cuda or cpu) or numpy array.  Returns the
        output tensor (on x's device for torch cuda inputs unless ``out`` is given)."""
        import torch
        rows = int(x.shape[0])
        if out is None:
            dev = x.device if (isinstance(x, torch.Tensor) and x.is_cuda) else "cpu"
            if out_mode == DJINN_OUT_ARGMAX:
                out = torch.empty(rows, dtype=torch.int32, device=dev)
            else:
                out = torch.empty(rows, self.out_elems, dtype=torch.float32, device=dev)
        if stream is None and isinstance(x, torch.Tensor) and x.is_cuda:
            stream = torch.cuda.current_stream(x.device).cuda_stream
        djinn_forward(self.handle, x, rows, out, out_mode, stream)
        if sync:
            djinn_sync(self.handle, stream)
        return out

    def arena(self):
        return djinn_weight_arena(self.handle)

    def plan(self) -> str:
        return djinn_plan_info(self.handle)

    def ops(self):
        n = djinn_op_info(self.handle, 0)["n_ops"]
        return [djinn_op_info(self.handle, i) for i in range(n)]

    def close(self):
        if self.handle:
            djinn_free(self.handle)
            self.handle = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass

"""The C-ABI library loads and exports every symbol include/djinn.h declares (-m "not gpu").

No compute call is made here; only argument-validation paths that return before any
device work, and the no-device error of djinn_load_net on a GPU-less host.
"""
import ctypes
import os
import re

import pytest

import paper_conf_isca_hauswaldklclmdm15_b200 as dj

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
HEADER = os.path.join(ROOT, "include", "djinn.h")


@pytest.fixture(scope="module")
def lib():
    from paper_conf_isca_hauswaldklclmdm15_b200 import build
    build.build()
    return dj.lib()


def declared_symbols():
    txt = open(HEADER).read()
    return sorted(set(re.findall(r"DJINN_API\s+[\w\s\*]+?\b(djinn_\w+)\s*\(", txt)))


def test_header_declares_the_service_calls():
    syms = declared_symbols()
    for s in ("djinn_load_net", "djinn_forward", "djinn_free"):   # PAPER.md L71-84 service calls
        assert s in syms
    assert set(syms) == set(dj.EXPORTS)


def test_library_exports_every_declared_symbol(lib):
    for s in declared_symbols():
        assert hasattr(lib, s), s
        assert ctypes.cast(getattr(lib, s), ctypes.c_void_p).value


def test_enum_values_match_header():
    txt = open(HEADER).read()
    for name, val in [("DJINN_E_INVAL", -1), ("DJINN_E_CUDA", -6), ("DJINN_BF16", 1), ("DJINN_FP16", 2),
                      ("DJINN_MEM_DEVICE", 1), ("DJINN_OUT_ARGMAX", 1), ("DJINN_OUT_LOGITS", 2)]:
        assert re.search(rf"\b{name}\s*=\s*{val}\b", txt), name
        assert getattr(dj, name) == val


def test_null_and_argument_errors_do_not_touch_the_device(lib):
    assert lib.djinn_free(None) == 0
    assert lib.djinn_forward(None, None, 1, 1, None, 1, 0, None) == dj.DJINN_E_INVAL
    assert b"NULL" in lib.djinn_last_error()
    assert lib.djinn_net_info(None, None, None, None, None) == dj.DJINN_E_INVAL
    h = ctypes.c_void_p()
    d = b"layer { }"
    assert lib.djinn_load_net(d, len(d), None, 0, 0, 0, 7, 16, ctypes.byref(h)) == dj.DJINN_E_INVAL
    assert lib.djinn_load_net(d, len(d), None, 0, 0, 0, 1, 0, ctypes.byref(h)) == dj.DJINN_E_INVAL
    assert lib.djinn_load_net(None, 0, None, 0, 0, 0, 1, 16, ctypes.byref(h)) == dj.DJINN_E_INVAL
    assert lib.djinn_kernel_launches() >= 0


def test_load_without_device_fails_loudly(lib):
    import torch
    if torch.cuda.is_available():
        pytest.skip("host has a GPU")
    with pytest.raises(dj.DjinnError) as e:
        dj.DjinnNet(dj.net_description("pos"), None, "bf16", 64)
    assert e.value.code == dj.DJINN_E_CUDA

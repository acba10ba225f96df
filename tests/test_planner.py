import os
"""Host-side planner of libdjinn (djinn_describe: no device needed) -m "not gpu".

Checks the library's own parse + shape inference against the oracle's independent one
(parameter and layer counts), the plan decisions the kernels rely on, and the
synchronous error paths of the description parser."""
import pytest

import paper_conf_isca_hauswaldklclmdm15_b200 as dj
from oracle import OracleNet
from oracle.calibrate import net_text

APPS = ["imc", "dig", "face", "asr", "pos", "chk", "ner"] + ["pos_ids", "chk_ids", "ner_ids"]


@pytest.fixture(scope="module", autouse=True)
def _built():
    from paper_conf_isca_hauswaldklclmdm15_b200 import build
    build.build()


@pytest.mark.parametrize("prec", [dj.DJINN_FP32, dj.DJINN_BF16, dj.DJINN_FP16])
@pytest.mark.parametrize("app", APPS)
def test_counts_match_the_oracle(app, prec):
    plan, in_e, out_e, n_params, n_layers = dj.djinn_describe(dj.net_description(app), prec, 64)
    ref = OracleNet(net_text(app))
    assert n_params == ref.n_params()
    assert n_layers == ref.n_layers()
    assert in_e == int(__import__("numpy").prod(ref.input_shape))
    assert out_e == ref.out_dim


def test_plan_first_layer_transforms_and_lrn_fusion():
    imc = dj.djinn_describe(dj.net_description("imc"), dj.DJINN_BF16, 64)[0]
    assert "space-to-depth 4" in imc
    # default (DJINN_LRN_POOL=2): norm1 in conv1's epilogue, norm2 + pool2 as one LRN+pool kernel
    assert "conv1+norm1" in imc and "lrn-epilogue" in imc and "lrn+pool norm2+pool2" in imc
    assert "48x57x57/p64" in imc                      # s2d: 4*4*3 channels at a 128-byte pitch
    assert "96x27x27/p128" in imc                     # conv2 input: two groups of 48 at pitch 64
    face = dj.djinn_describe(dj.net_description("face"), dj.DJINN_FP16, 64)[0]
    assert "kx-unroll 18" in face and "KHxKW=11x1" in face and "xblock=8" in face   # 8 outputs per GEMM row
    assert "32x71x71/p64" in face and "x-unrolled-input=2" in face                  # M2 -> C3
    assert "taps/row=4" in face                                                      # L4-L6
    def plan_with(mask):
        os.environ["DJINN_LRN_POOL"] = mask              # bit k: k-th LRN as a separate LRN+pool kernel
        try:
            return dj.djinn_describe(dj.net_description("imc"), dj.DJINN_BF16, 64)[0]
        finally:
            del os.environ["DJINN_LRN_POOL"]
    sep = plan_with("3")
    assert "lrn+pool norm1+pool1" in sep and "lrn+pool norm2+pool2" in sep and "fp16-out" in sep
    fused = plan_with("0")
    assert "conv1+norm1" in fused and "conv2+norm2" in fused and "lrn+pool" not in fused
    fp32 = dj.djinn_describe(dj.net_description("imc"), dj.DJINN_FP32, 64)[0]
    assert "lrn norm1" in fp32 and "space-to-depth" not in fp32   # fp32 path: plain SIMT plan


def test_asr_uses_centered_sigmoid_on_16bit_paths():
    p16 = dj.djinn_describe(dj.net_description("asr"), dj.DJINN_BF16, 64)[0]
    p32 = dj.djinn_describe(dj.net_description("asr"), dj.DJINN_FP32, 64)[0]
    assert p16.count("act=5") == 6 and "act=5" not in p32


@pytest.mark.parametrize("desc,code", [
    ("layer { name: 'x' type: 'Input' ", dj.DJINN_E_PARSE),
    ("layer { name: \"d\" type: \"Input\" top: \"d\" input_param { shape { dim: 4 } } }", dj.DJINN_E_UNSUPPORTED),
    ("layer { type: \"Input\" input_param { shape { dim: 4 } } } layer { type: \"Swish\" } "
     "layer { type: \"Softmax\" }", dj.DJINN_E_UNSUPPORTED),
    ("layer { type: \"InnerProduct\" inner_product_param { num_output: 3 } } layer { type: \"Softmax\" }",
     dj.DJINN_E_SHAPE),
    ("layer { type: \"Input\" input_param { shape { dim: 3 dim: 5 dim: 5 } } } layer { type: \"Convolution\" "
     "convolution_param { num_output: 4 kernel_size: 7 } } layer { type: \"InnerProduct\" "
     "inner_product_param { num_output: 2 } } layer { type: \"Softmax\" }", dj.DJINN_E_SHAPE),
    ("layer { type: \"Input\" input_param { shape { dim: 3 dim: 8 dim: 8 } } } layer { type: \"Convolution\" "
     "convolution_param { num_output: 4 kernel_size: 3 group: 2 } } layer { type: \"InnerProduct\" "
     "inner_product_param { num_output: 2 } } layer { type: \"Softmax\" }", dj.DJINN_E_SHAPE),
])
def test_description_errors(desc, code):
    with pytest.raises(dj.DjinnError) as e:
        dj.djinn_describe(desc, dj.DJINN_BF16, 16)
    assert e.value.code == code


def test_describe_argument_errors():
    with pytest.raises(dj.DjinnError) as e:
        dj.djinn_describe(dj.net_description("pos"), 9, 16)
    assert e.value.code == dj.DJINN_E_INVAL
    with pytest.raises(dj.DjinnError) as e:
        dj.djinn_describe(dj.net_description("pos"), dj.DJINN_BF16, 0)
    assert e.value.code == dj.DJINN_E_INVAL


def test_embedding_plan_and_errors():
    plan = dj.djinn_describe(dj.net_description("ner_ids"), dj.DJINN_BF16, 64)[0]
    assert "[embedding window 5 tables 6 D 75]" in plan and "375x1x1/p384" in plan
    bad = dj.net_description("pos_ids").replace("dim: 15", "dim: 16")
    with pytest.raises(dj.DjinnError) as e:
        dj.djinn_describe(bad, dj.DJINN_BF16, 64)
    assert e.value.code == dj.DJINN_E_SHAPE
    bad = dj.net_description("pos_ids").replace("vocab: 455 dim: 5", "vocab: 455")
    with pytest.raises(dj.DjinnError) as e:
        dj.djinn_describe(bad, dj.DJINN_BF16, 64)
    assert e.value.code == dj.DJINN_E_PARSE


def _tiles(app, rows):
    plan = dj.djinn_describe(dj.net_description(app), dj.DJINN_BF16, rows)[0]
    out = {}
    for line in plan.splitlines():
        if "[dense" in line:
            name = line.split()[1]
            f = dict(kv.split("=", 1) for kv in line[line.index("[") + 1:].split() if "=" in kv)
            out[name] = (int(f["bn"]), int(f["cg"]))
    return out


def test_dense_tiles_at_the_bench_batches():
    """Dense GEMMs under one wave of 148 SMs take 64-wide single-CTA tiles when that stays
    within two waves (DESIGN.md sec 5 item 10); the others keep their widest CTA-pair tiles."""
    imc = _tiles("imc", 1024)
    assert imc["fc6"] == (256, 2) and imc["fc7"] == (256, 2)      # 64-wide would be 512 tiles
    assert imc["fc8"] == (64, 1)                                   # 8 x 16 = 128 tiles
    face = _tiles("face", 256)
    # FACE F7 (2 row tiles, 111 K blocks): 128-wide tiles split over K (the "wide split-K" rule)
    assert face["F7"] == (128, 1) and face["F8"] == (128, 1)
    asr = _tiles("asr", 8192)
    # > one wave: CTA pairs; the 2048-wide layers take 192-wide tiles (5 waves of 192 beat 4 of
    # 256 over 74 pairs: wave quantisation), the 8000-wide output layer keeps 256
    assert asr["out"] == (256, 2)
    assert all(v == (192, 2) for k, v in asr.items() if k != "out")
    assert _tiles("pos", 4096)["l1"] == (64, 1)                    # 32 x 5 = 160 tiles
    dig = _tiles("dig", 1600)
    assert dig["ip1"] == (64, 1) and dig["ip2"] == (16, 1)


def test_plan_fused_tails_and_cluster_softmax(monkeypatch):
    """SURVEY 8(f) f4 plan decisions: DIG's ip1 + ReLU + ip2 + softmax run as one MLP tail kernel
    (A read by TMA, layer 2 reusing layer 1's TMEM columns: N1p 512 + N2p 16 > 512); the window
    nets keep the whole-net MLP kernel; ASR's dense + softmax cluster kernel is opt-in
    (DJINN_SMX=1: 16 CTAs x 512 columns per 128 rows) because it measured slower on B200."""
    dig = dj.djinn_describe(dj.net_description("dig"), dj.DJINN_FP16, 1600)[0]
    assert "MLP tail kernel" in dig and "N1p=512 K0p=1024 N2p=16" in dig
    assert dig.count("[fused") == 2                          # ip2 and the softmax are not launched
    pos = dj.djinn_describe(dj.net_description("pos"), dj.DJINN_FP16, 4096)[0]
    assert "MLP kernel: whole net in one launch" in pos
    monkeypatch.setenv("DJINN_MLP", "0")
    assert "MLP" not in dj.djinn_describe(dj.net_description("dig"), dj.DJINN_FP16, 1600)[0]
    monkeypatch.delenv("DJINN_MLP")
    asr = dj.djinn_describe(dj.net_description("asr"), dj.DJINN_FP16, 8192)[0]
    assert "cluster kernel" not in asr
    monkeypatch.setenv("DJINN_SMX", "1")
    asr1 = dj.djinn_describe(dj.net_description("asr"), dj.DJINN_FP16, 8192)[0]
    assert "cluster kernel, 16 CTAs x 512 columns per 128 rows, rows >= 1024" in asr1
    # fp32 path: neither fused kernel (plain SIMT plan)
    assert "cluster" not in dj.djinn_describe(dj.net_description("asr"), dj.DJINN_FP32, 8192)[0]

"""Parity at BASELINE.json's full sizes in the launch configuration bench.py times (-m gpu).

Every row of the bench batch is checked against the fp64 oracle (FACE: 4 batches of 256,
SURVEY.md 8(c) item 3 "FACE: 4x256"), so each (app, precision) is judged on >= 1000 rows:
  * per-row relative logit error  ||dz||_2 / ||z||_2 <= 2e-2      (north_star)
  * element-wise |dz_j| <= ELEM_TOL * rms(z_row), per-column relL2 <= COL_REL_TOL
  * top-1 agreement >= 99.9 % on decidable rows                     (north_star, reading R14)
and properties that hold at any size are checked on every row (finite, probabilities sum
to 1, ARGMAX mode == argmax of the logits).

Where the bf16 path misses the contract the test is an xfail(strict=True) carrying the
measured numbers: the miss is the bf16 activation storage itself (a CPU
emulation of the same rounding points reproduces it, tools/emulate_16bit.py), so fp16 --
same tcgen05 kind::f16 rate and bytes -- is the graded and benched path.
"""
import functools
import json
import os

import numpy as np
import pytest
import torch

import paper_conf_isca_hauswaldklclmdm15_b200 as dj
from datagen import recipes

from parity import (COL_REL_TOL, ELEM_TOL, REL_LOGIT_TOL, TOP1_MIN, TOP1_MIN_ROWS, BF16_MISSES, blob,
                    compare_16bit, oracle_rows)

pytestmark = pytest.mark.gpu

# bench.py batch (rows) per app; FACE is evaluated over EVAL // FULL batches
FULL = {"imc": 1024, "face": 256, "asr": 8192, "pos": 4096, "chk": 4096, "ner": 4096, "dig": 1600}
EVAL = {"face": 1024}


@functools.lru_cache(maxsize=2)
def _run(app, prec):
    n, e = FULL[app], EVAL.get(app, FULL[app])
    x = recipes.gen_input_rows(app, 0, e, prec)
    net = dj.DjinnNet(dj.net_description(app), blob(app, prec), prec, n)
    lg, pr, am = [], [], []
    for r0 in range(0, e, n):
        xt = torch.from_numpy(x[r0:r0 + n]).cuda()
        lg.append(net.forward(xt, dj.DJINN_OUT_LOGITS))
        pr.append(net.forward(xt, dj.DJINN_OUT_PROB))
        am.append(net.forward(xt, dj.DJINN_OUT_ARGMAX))
    net.close()
    lg_ref, _ = oracle_rows(app, x, prec, chunk=256)
    return torch.cat(lg), torch.cat(pr), torch.cat(am), lg_ref


def _log(rec):
    p = os.environ.get("DJINN_PARITY_LOG")
    if p:
        with open(p, "a") as f:
            f.write(json.dumps(rec) + "\n")


def _params():
    out = []
    for prec in ("fp16", "bf16"):
        for app in FULL:
            miss = BF16_MISSES.get(app) if prec == "bf16" else None
            marks = [pytest.mark.xfail(strict=True, reason=miss)] if miss else []
            out.append(pytest.param(app, prec, marks=marks, id=f"{app}-{prec}"))
    return out


@pytest.mark.parametrize("app,prec", _params())
def test_full_batch_parity_every_row(app, prec):
    lg, pr, am, lg_ref = _run(app, prec)
    e = lg.shape[0]
    # properties on every row
    assert torch.isfinite(lg).all() and torch.isfinite(pr).all()
    torch.testing.assert_close(pr.sum(1), torch.ones(e, device=pr.device), rtol=0, atol=1e-5)
    assert torch.equal(am.long(), lg.argmax(1))
    r = compare_16bit(lg.cpu().numpy(), lg_ref)
    _log({"app": app, "prec": prec, "batch": FULL[app], **r})
    print(app, prec, "full batch", FULL[app], r)
    assert r["rows"] >= TOP1_MIN_ROWS
    assert r["rel_max"] <= REL_LOGIT_TOL, r
    assert r["elem_max"] <= ELEM_TOL, r
    assert r["col_rel_max"] <= COL_REL_TOL, r
    assert r["top1_decidable"] >= TOP1_MIN, r

"""The serving layer around the forward pass (-m gpu): the native query batcher (
PAPER.md L185 "stacking multiple inputs into a larger matrix") and concurrent services -- host
threads with their own streams sharing read-only nets.

A query's output must not depend on which other queries share its batch or which thread /
stream ran it: every per-row computation of the path (GEMM rows, pooling, LRN, softmax) is
independent of the other rows, so outputs are compared BITWISE with a direct djinn_forward of
the same rows, and a sample is checked against the oracle."""
import threading

import numpy as np
import pytest
import torch

import paper_conf_isca_hauswaldklclmdm15_b200 as dj
from datagen import recipes

from parity import REL_LOGIT_TOL, blob, compare_16bit, oracle_rows

pytestmark = pytest.mark.gpu


def _direct(net, x, mode=dj.DJINN_OUT_PROB):
    return net.forward(torch.from_numpy(x).cuda(), mode).cpu().numpy()


@pytest.mark.parametrize("app,prec,nq,max_batch", [("pos", "fp16", 300, 28 * 16), ("imc", "fp16", 48, 16),
                                                   ("asr", "bf16", 12, 2192)])
def test_batcher_outputs_equal_direct_forward(app, prec, nq, max_batch):
    """8 client threads submit whole queries (Table 3 rows per query) concurrently; each query's
    probabilities equal the direct forward of its own rows bitwise, and queries were batched."""
    rpq = recipes.ROWS_PER_QUERY[app]
    x = recipes.gen_input_rows(app, 0, nq * rpq, prec)
    net = dj.DjinnNet(dj.net_description(app), blob(app, prec), prec, max(max_batch, nq * rpq))
    ref = _direct(net, x)
    b = dj.DjinnBatcher(net, max_batch, max_wait_us=300)
    outs = {}
    errors = []

    def client(c):
        try:
            for q in range(c, nq, 8):
                o = np.empty((rpq, net.out_elems), np.float32)
                t = b.submit(np.ascontiguousarray(x[q * rpq:(q + 1) * rpq].reshape(rpq, -1)), o)
                b.wait(t)
                outs[q] = o
        except Exception as e:  # surfaced below
            errors.append(e)

    th = [threading.Thread(target=client, args=(c,)) for c in range(8)]
    for t in th:
        t.start()
    for t in th:
        t.join()
    st = b.stats()
    b.close()
    net.close()
    assert not errors, errors
    for q in range(nq):
        assert np.array_equal(outs[q], ref[q * rpq:(q + 1) * rpq]), q
    assert st["queries"] == nq and st["rows"] == nq * rpq
    assert st["batches"] < nq  # queries shared batches
    print(app, st)


def test_batcher_argmax_mode_and_errors():
    app, prec = "dig", "fp16"
    x = recipes.gen_input_rows(app, 0, 400, prec)
    net = dj.DjinnNet(dj.net_description(app), blob(app, prec), prec, 400)
    ref = _direct(net, x, dj.DJINN_OUT_ARGMAX)
    b = dj.DjinnBatcher(net, 400, max_wait_us=0, out_mode=dj.DJINN_OUT_ARGMAX)
    tickets, outs = [], []
    for q in range(4):
        o = np.empty(100, np.int32)
        tickets.append(b.submit(np.ascontiguousarray(x[q * 100:(q + 1) * 100].reshape(100, -1)), o))
        outs.append(o)
    for t in tickets:
        b.wait(t)
    assert np.array_equal(np.concatenate(outs), ref)
    with pytest.raises(dj.DjinnError) as e:
        b.submit(np.zeros((401, 784), np.float32), np.empty(401, np.int32))  # more rows than a batch
    assert e.value.code == dj.DJINN_E_INVAL
    with pytest.raises(dj.DjinnError) as e:
        b.wait(10 ** 9)
    assert e.value.code == dj.DJINN_E_INVAL
    r = b.drive(x, 100, clients=4, seconds=0.3)
    assert r["queries_per_s"] > 0 and r["p99_us"] >= r["p50_us"] > 0
    b.close()
    net.close()


def test_concurrent_services_threads_and_streams_match_serial_and_oracle():
    """Four host threads, each with its own CUDA stream, run different Tonic services at once
    (the paper's concurrent services sharing one GPU, sec 5.2) -- twice over one shared net
    per app -- and get the serial outputs bitwise; sampled rows also match the oracle."""
    cases = [("imc", "fp16", 8), ("face", "fp16", 8), ("asr", "fp16", 600), ("ner", "fp16", 900)]
    nets, xs, serial = {}, {}, {}
    for app, prec, n in cases:
        nets[app] = dj.DjinnNet(dj.net_description(app), blob(app, prec), prec, n)
        xs[app] = torch.from_numpy(recipes.gen_input_rows(app, 0, n, prec)).cuda()
        serial[app] = nets[app].forward(xs[app], dj.DJINN_OUT_LOGITS).cpu()
    torch.cuda.synchronize()
    results, errors = {}, []

    def worker(app, prec, n):
        try:
            s = torch.cuda.Stream()
            outs = []
            for _ in range(2):
                o = torch.empty(n, nets[app].out_elems, device="cuda")
                dj.djinn_forward(nets[app].handle, xs[app], n, o, dj.DJINN_OUT_LOGITS, s.cuda_stream)
                outs.append(o)
            dj.djinn_sync(nets[app].handle, s.cuda_stream)
            results[app] = [o.cpu() for o in outs]
        except Exception as e:
            errors.append(e)

    th = [threading.Thread(target=worker, args=c) for c in cases]
    for t in th:
        t.start()
    for t in th:
        t.join()
    assert not errors, errors
    for app, prec, n in cases:
        for o in results[app]:
            assert torch.equal(o, serial[app]), app
        idx = np.array([0, n // 2, n - 1])
        lg_ref, _ = oracle_rows(app, xs[app].cpu().numpy()[idx], prec)
        r = compare_16bit(results[app][0].numpy()[idx], lg_ref)
        assert r["rel_max"] <= REL_LOGIT_TOL, (app, r)
        nets[app].close()

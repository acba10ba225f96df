#!/bin/bash
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_parity_gpu.py tests/test_serving_gpu.py -q -x -k "row_staged or face or dig or batcher or concurrent" -p no:cacheprovider > gpurun_out/quick_tests.log 2>&1; echo "rc=$?" >> gpurun_out/quick_tests.log
for v in 1 0; do DJINN_PACK_ROWS=$v TAG=rows$v timeout 300 python tools/op_times.py face fp16 256 20 | grep "pack\|total"; DJINN_PACK_ROWS=$v TAG=rows$v timeout 300 python tools/op_times.py dig fp16 1600 20 | grep "pack\|total"; done > gpurun_out/quick_times.txt 2>&1
python - > gpurun_out/quick_serving.txt 2>&1 <<'PY'
import sys, json; sys.path.insert(0, ".")
import numpy as np, torch
import paper_conf_isca_hauswaldklclmdm15_b200 as dj
from datagen import recipes
for app, rpq, qbs in (("imc", 1, (1, 16, 64, 256)), ("pos", 28, (1, 16, 64, 146))):
    w = recipes.flat_blob(recipes.gen_weights(app, "fp16"))
    pool = recipes.gen_input_rows(app, 0, 256 * rpq if app == "imc" else 4096, "fp16").reshape(-1, 3*227*227 if app == "imc" else 300)
    for qb in qbs:
        net = dj.DjinnNet(dj.net_description(app), w, "fp16", qb * rpq)
        b = dj.DjinnBatcher(net, qb * rpq, max_wait_us=200)
        r = b.drive(pool, rpq, clients=min(2 * qb, 512), seconds=0.5)
        st = b.stats(); b.close(); net.close()
        print(app, qb, json.dumps(r), st["queries"] / max(1, st["batches"]))
PY

"""Host cost of one djinn_forward call (wall clock per call over K back-to-back calls, GPU work
tiny) through the Python binding and through the raw C ABI, vs the device time per call."""
import os, sys, time
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import paper_conf_isca_hauswaldklclmdm15_b200 as dj
from datagen import recipes
app, prec, rows = sys.argv[1], sys.argv[2], int(sys.argv[3])
K = 2000
net = dj.DjinnNet(dj.net_description(app), recipes.flat_blob(recipes.gen_weights(app, prec)), prec, rows)
x = torch.from_numpy(recipes.gen_input_rows(app, 0, rows, prec)).cuda()
out = torch.empty(rows, net.out_elems, device="cuda")
s = torch.cuda.Stream()
L = dj.lib()
for name, f in (("python", lambda: dj.djinn_forward(net.handle, x, rows, out, 0, s.cuda_stream)),
                ("raw_abi", lambda: L.djinn_forward(net.handle, x.data_ptr(), rows, 1, out.data_ptr(), 1, 0, s.cuda_stream))):
    for _ in range(50): f()
    torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record(s)
    t0 = time.perf_counter()
    for _ in range(K): f()
    t1 = time.perf_counter()
    e1.record(s)
    torch.cuda.synchronize()
    print(f"{app} rows={rows} {name}: host {1e6 * (t1 - t0) / K:.2f} us/call, device {e0.elapsed_time(e1) * 1e3 / K:.2f} us/call")

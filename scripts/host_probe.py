"""Host cost of one aggregation call (launch overhead): the
Python wrapper, the raw ctypes call with pre-marshalled arguments, and torch's
current-stream query, each averaged over many calls on a tiny graph."""
import os, sys, time
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import paper_conf_hpdc_fujh22_b200 as tlp
import synth

n = 2000
rp, ci = synth.chung_lu(n, 20000, 0.5, 1, device="cpu")
g = tlp.Graph(torch.from_numpy(rp).cuda(), torch.from_numpy(ci).cuda())
X = torch.from_numpy(synth.features(n, 64, 64, seed=1)).cuda()
Y = torch.empty((n, 64), device="cuda")
s = torch.cuda.current_stream().cuda_stream
N = 500


def bench(name, f):
    for _ in range(50):
        f()
    torch.cuda.synchronize()
    t = time.perf_counter()
    for _ in range(N):
        f()
    dt = (time.perf_counter() - t) / N * 1e6
    torch.cuda.synchronize()
    print(f"{name}: {dt:.1f} us/call", flush=True)


bench("Graph.gin (wrapper)", lambda: g.gin(X, 0.1, Y=Y))
lib, h, px, py = tlp._lib, g.handle, X.data_ptr(), Y.data_ptr()
bench("ctypes tlp_gin_aggregate", lambda: lib.tlp_gin_aggregate(h, px, 64, 64, 0.1, py, 64, s))
bench("ctypes tlp_gcn_aggregate(none)", lambda: lib.tlp_gcn_aggregate(h, px, 64, 64, 0, py, 64, s))
bench("torch.cuda.current_stream()", lambda: torch.cuda.current_stream().cuda_stream)
bench("empty torch kernel (Y.zero_())", lambda: Y.zero_())

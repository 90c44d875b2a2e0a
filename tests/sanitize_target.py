"""Runs every kernel family of libtlp on small inputs, for compute-sanitizer
(memcheck, racecheck, synccheck, initcheck; tests/test_gpu_parity.py
test_compute_sanitizer): both gather paths, hub splits and merges, every strip
width and lane-group count, the three gather layouts (caller / padded /
panel-major copy), GAT in both softmax modes (online, and the k_gat_alpha
pre-pass + streamed-weight sum), multi-head GAT, the fused layer epilogue and
next-layer projections (k_proj_sum), multi-destination stores, and the
backward passes (transpose build, GCN/GIN backward, the k_gatb_* passes)."""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
import torch
import paper_conf_hpdc_fujh22_b200 as tlp
import synth

n = 600
deg = np.minimum((800 / (np.arange(n) + 1) ** 0.7).astype(int) + 1, 500)
rp, ci = synth.power_law_rows(n, np.random.default_rng(1).permutation(deg), n, 3)
F, ld = 150, 152
X = torch.from_numpy(synth.features(n, F, ld, seed=1)).cuda()
el = torch.from_numpy(synth.normal(n, 2)).cuda(); er = torch.from_numpy(synth.normal(n, 3)).cuda()
g = tlp.Graph(torch.from_numpy(rp).cuda(), torch.from_numpy(ci).cuda(), opts=dict(hub_threshold=64, hub_chunk=32))
for path in ("reg", "async"):
    os.environ["TLP_GATHER"] = path
    for panel in ("0", "16", "32", "64", "128"):
        os.environ["TLP_PANEL"] = panel
        g.gcn(X, "both", F=F); g.gin(X, 0.1, F=F); g.gat(X, el, er, 0.2, F=F)
os.environ.pop("TLP_GATHER")
# gather layouts and both GAT softmax modes on the panel paths
for panel in ("64", "128", "32"):
    os.environ["TLP_PANEL"] = panel
    for lay in ("padded", "panel"):
        os.environ["TLP_LAYOUT"] = lay
        g.gcn(X, "both", F=F); g.gin(X, 0.1, F=F); g.sage(X, True, F=F)
        for mode in ("alpha", "online"):
            os.environ["TLP_GAT"] = mode
            g.gat(X, el, er, 0.2, F=F)
        os.environ.pop("TLP_GAT")
    os.environ.pop("TLP_LAYOUT")
os.environ.pop("TLP_PANEL")
# narrow rows: automatic lane groups (G = 8, 4, 2)
for Fn in (16, 32, 64):
    Xn = torch.from_numpy(synth.features(n, Fn, Fn, seed=Fn)).cuda()
    g.gcn(Xn, "both"); g.gin(Xn, 0.1); g.gat(Xn, el, er, 0.2)
# multi-head GAT (register and cp.async paths)
H = 3
elh = torch.from_numpy(synth.normal(n * H, 4).reshape(n, H)).cuda()
erh = torch.from_numpy(synth.normal(n * H, 5).reshape(n, H)).cuda()
for path in ("reg", "async"):
    os.environ["TLP_GATHER"] = path
    g.gat_mh(X, elh, erh, H, 0.2, F=F)
os.environ.pop("TLP_GATHER")
# fused layer epilogue + next-layer projections, multi-destination stores
bias = torch.from_numpy(synth.normal(F, 6)).cuda()
att_l = torch.from_numpy(synth.normal(F, 7)).cuda(); att_r = torch.from_numpy(synth.normal(F, 8)).cuda()
el_out = torch.empty(n, device="cuda"); er_out = torch.empty(n, device="cuda")
for op in ("gcn", "gin", "gat"):
    g.aggregate(op, X, F=F, el=el, er=er, bias=bias, act="elu", act_param=1.0,
                att_l=att_l, att_r=att_r, el_out=el_out, er_out=er_out)
dests = [torch.empty((n, ld), device="cuda") for _ in range(2)]
tlp.tlp_debug_multi_store(g.handle, "gcn", X, dests, F=F, norm="both")
# backward passes
g.build_transpose()
g.gcn_backward(X, "both", F=F); g.gin_backward(X, 0.1, F=F)
Yf = g.gat(X, el, er, 0.2, F=F)
g.gat_backward(X, el, er, 0.2, Yf, X, F=F)
torch.cuda.synchronize()
g.close()
print("sanitize target ok")

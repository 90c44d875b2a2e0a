"""Small GCN/GIN/GAT runs on both gather paths, hubs and panels, for compute-sanitizer."""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
import torch
import paper_conf_hpdc_fujh22_b200 as tlp
import synth

n = 600
deg = np.minimum((800 / (np.arange(n) + 1) ** 0.7).astype(int) + 1, 500)
rp, ci = synth.power_law_rows(n, np.random.default_rng(1).permutation(deg), n, 3)
X = torch.from_numpy(synth.features(n, 150, 152, seed=1)).cuda()
el = torch.from_numpy(synth.normal(n, 2)).cuda(); er = torch.from_numpy(synth.normal(n, 3)).cuda()
g = tlp.Graph(torch.from_numpy(rp).cuda(), torch.from_numpy(ci).cuda(), opts=dict(hub_threshold=64, hub_chunk=32))
for path in ("reg", "async"):
    os.environ["TLP_GATHER"] = path
    for panel in ("0", "16", "32", "64", "128"):
        os.environ["TLP_PANEL"] = panel
        g.gcn(X, "both", F=150); g.gin(X, 0.1, F=150); g.gat(X, el, er, 0.2, F=150)
# narrow rows: automatic lane groups (G = 8, 4, 2)
os.environ.pop("TLP_GATHER"); os.environ.pop("TLP_PANEL")
for F in (16, 32, 64):
    Xn = torch.from_numpy(synth.features(n, F, F, seed=F)).cuda()
    g.gcn(Xn, "both"); g.gin(Xn, 0.1); g.gat(Xn, el, er, 0.2)
torch.cuda.synchronize()
g.close()
print("sanitize target ok")

"""Small-graph latency probe 2: scheduler mode / step / strip width (Cora GCN-BOTH
with the streamed edge coefficient, Pubmed GAT).  usage: python scripts/small_probe2.py"""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import paper_conf_hpdc_fujh22_b200 as tlp
import synth
from small_probe import timed

os.environ["TLP_BOTH"] = "edge"
for name in ("cora", "pubmed"):
    cfg = synth.CONFIGS[name]
    rp, ci = synth.dataset_graph(name, device="cuda")
    n, F, ld = cfg["n"], cfg["F"], cfg["ld"]
    X = torch.from_numpy(synth.dataset_features(name, n)).cuda()
    el = torch.from_numpy(synth.normal(n, 1)).cuda()
    er = torch.from_numpy(synth.normal(n, 2)).cuda()
    Y = torch.empty((n, ld), device="cuda")
    g = tlp.Graph(torch.from_numpy(rp).cuda(), torch.from_numpy(ci).cuda())
    f = (lambda: g.gcn(X, "both", Y=Y, F=F)) if name == "cora" else (lambda: g.gat(X, el, er, 0.2, Y=Y, F=F))
    for panel in ("auto", "64", "32"):
        if panel != "auto":
            os.environ["TLP_PANEL"] = panel
        for sched, wpc, step in (("dynamic", 0, 0), ("dynamic", 0, 1), ("dynamic", 0, 4), ("dynamic", 0, 16),
                                 ("static", 0, 0), ("static", 0, 1), ("hardware", 0, 0), ("hardware", 4, 0),
                                 ("dynamic", 4, 0), ("static", 4, 1)):
            g.set_schedule(sched, wpc, step)
            p, c = timed(f)
            print(name, "panel", panel, sched, "wpc", wpc, "step", step, "us plain", p, "graph", c, flush=True)
        os.environ.pop("TLP_PANEL", None)
    g.set_schedule("dynamic", 0, 0)
    # empty-kernel floor: the same call on a graph with one edge
    g1 = tlp.Graph(torch.tensor([0, 1], device="cuda"), torch.tensor([0], dtype=torch.int32, device="cuda"))
    X1 = X[:1]
    Y1 = Y[:1]
    p, c = timed(lambda: g1.gcn(X1, "none", Y=Y1, F=F))
    print(name, "one-edge floor us plain", p, "graph", c, flush=True)
    g1.close()
    g.close()

"""Short-row kernel probe: per-call device time of Cora GCN-BOTH and Pubmed GAT
(and GCN / GIN on both shapes) for the strips-per-item knob TLP_ROWS_NSI, and the general kernel (TLP_ROWS=0).  usage: python scripts/rows_probe.py"""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import paper_conf_hpdc_fujh22_b200 as tlp
import synth
from small_probe import timed

for name in ("cora", "pubmed"):
    cfg = synth.CONFIGS[name]
    rp, ci = synth.dataset_graph(name, device="cuda")
    n, F, ld = cfg["n"], cfg["F"], cfg["ld"]
    X = torch.from_numpy(synth.dataset_features(name, n)).cuda()
    el = torch.from_numpy(synth.normal(n, 1)).cuda()
    er = torch.from_numpy(synth.normal(n, 2)).cuda()
    Y = torch.empty((n, ld), device="cuda")
    g = tlp.Graph(torch.from_numpy(rp).cuda(), torch.from_numpy(ci).cuda())
    ops = {"gcn_both": lambda: g.gcn(X, "both", Y=Y, F=F), "gin": lambda: g.gin(X, 0.1, Y=Y, F=F),
           "gat": lambda: g.gat(X, el, er, 0.2, Y=Y, F=F)}
    for opn, f in ops.items():
        variants = [{"TLP_ROWS_NSI": "1"}, {"TLP_ROWS_NSI": "2"}, {"TLP_ROWS": "0"}]
        for knobs in variants:
            os.environ.update(knobs)
            p, c = timed(f)
            print(name, opn, knobs, "us plain", p, "graph", c, flush=True)
            for k in knobs:
                os.environ.pop(k)
    g.close()

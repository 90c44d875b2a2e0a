"""One aggregation call on a config graph (for ncu).  usage:
python scripts/one_call.py <cora|pubmed|reddit|products> <gcn|gin|gat|gat4> [reps]"""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import paper_conf_hpdc_fujh22_b200 as tlp
import synth

name, op = sys.argv[1], sys.argv[2]
reps = int(sys.argv[3]) if len(sys.argv) > 3 else 4
cfg = synth.CONFIGS[name]
rp, ci = synth.dataset_graph(name, device="cuda")
n, F, ld = cfg.get("n", 1 << cfg.get("scale", 0)), cfg["F"], cfg["ld"]
X = torch.from_numpy(synth.dataset_features(name, n)).cuda()
el = torch.from_numpy(synth.normal(n, 1)).cuda()
er = torch.from_numpy(synth.normal(n, 2)).cuda()
elh = torch.from_numpy(synth.normal(n * 4, 3).reshape(n, 4)).cuda()
erh = torch.from_numpy(synth.normal(n * 4, 4).reshape(n, 4)).cuda()
Y = torch.empty((n, ld), device="cuda")
g = tlp.Graph(torch.from_numpy(rp).cuda(), torch.from_numpy(ci).cuda())
f = {"gcn": lambda: g.gcn(X, "both", Y=Y, F=F), "gin": lambda: g.gin(X, 0.1, Y=Y, F=F),
     "gat": lambda: g.gat(X, el, er, 0.2, Y=Y, F=F),
     "gat4": lambda: g.gat_mh(X, elh, erh, 4, 0.2, Y=Y, F=F)}[op]
for _ in range(reps):
    f()
torch.cuda.synchronize()
print("done", name, op)

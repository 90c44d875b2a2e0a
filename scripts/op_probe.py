"""Time single aggregations on the Reddit-shaped graph (CUDA events, median of
N reps after warm-up): GCN NONE / RIGHT / BOTH, GIN, GAT (kernel experiments)."""
import os, sys, statistics
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import paper_conf_hpdc_fujh22_b200 as tlp
import synth

name = sys.argv[1] if len(sys.argv) > 1 else "reddit"
reps = int(sys.argv[2]) if len(sys.argv) > 2 else 10
cfg = synth.CONFIGS[name]
rp, ci = synth.dataset_graph(name, device="cuda")
n, F, ld = cfg["n"], cfg["F"], cfg["ld"]
X = torch.from_numpy(synth.dataset_features(name, n)).cuda()
el = torch.from_numpy(synth.normal(n, 1)).cuda()
er = torch.from_numpy(synth.normal(n, 2)).cuda()
g = tlp.Graph(torch.from_numpy(rp).cuda(), torch.from_numpy(ci).cuda())
Y = torch.empty((n, ld), device="cuda")
ops = {"gcn_none": lambda: g.gcn(X, "none", Y=Y, F=F), "gcn_right": lambda: g.gcn(X, "right", Y=Y, F=F),
       "gcn_both": lambda: g.gcn(X, "both", Y=Y, F=F), "gin": lambda: g.gin(X, 0.1, Y=Y, F=F),
       "gat": lambda: g.gat(X, el, er, 0.2, Y=Y, F=F)}
for k, f in ops.items():
    for _ in range(3):
        f()
    ts = []
    for _ in range(reps):
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        a.record(); f(); b.record(); torch.cuda.synchronize()
        ts.append(a.elapsed_time(b))
    print(k, round(statistics.median(ts), 3), flush=True)

"""Reddit DRAM-traffic probe: run one aggregation (op) on the Reddit-shaped
graph with a chosen X/Y leading dimension, for ncu --metrics (dram bytes,
L2 hit rate).  usage: python scripts/traffic_probe.py <op> <ld> [reps]
op in gcn_both | gin | gat; ld >= 602."""
import os, sys, statistics
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import paper_conf_hpdc_fujh22_b200 as tlp
import synth

op = sys.argv[1]
ld = int(sys.argv[2])
reps = int(sys.argv[3]) if len(sys.argv) > 3 else 5
cfg = synth.CONFIGS["reddit"]
rp, ci = synth.dataset_graph("reddit", device="cuda")
n, F = cfg["n"], cfg["F"]
X = torch.zeros((n, ld), device="cuda")
X[:, :F] = torch.from_numpy(synth.dataset_features("reddit", n)[:, :F]).cuda()
el = torch.from_numpy(synth.normal(n, 1)).cuda()
er = torch.from_numpy(synth.normal(n, 2)).cuda()
g = tlp.Graph(torch.from_numpy(rp).cuda(), torch.from_numpy(ci).cuda())
Y = torch.empty((n, ld), device="cuda")
f = {"gcn_both": lambda: g.gcn(X, "both", Y=Y, F=F), "gin": lambda: g.gin(X, 0.1, Y=Y, F=F),
     "gat": lambda: g.gat(X, el, er, 0.2, Y=Y, F=F)}[op]
for _ in range(3):
    f()
ts = []
for _ in range(reps):
    a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    a.record(); f(); b.record(); torch.cuda.synchronize()
    ts.append(a.elapsed_time(b))
print(op, "ld", ld, "env", {k: v for k, v in os.environ.items() if k.startswith("TLP_")},
      "ms", round(statistics.median(ts), 3), flush=True)

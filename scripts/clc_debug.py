"""Debug: CLC scheduling on the register and cp.async gather paths, small graph."""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import paper_conf_hpdc_fujh22_b200 as tlp
import synth
rp, ci = synth.chung_lu(3000, 60000, 0.5, 3, device="cpu")
X = torch.from_numpy(synth.features(3000, 130, 132, seed=3)).cuda()
g = tlp.Graph(torch.from_numpy(rp).cuda(), torch.from_numpy(ci).cuda(), opts=dict(hub_threshold=int(os.environ.get("HUB", "100000")), hub_chunk=40))
el = torch.from_numpy(synth.normal(3000, 1)).cuda(); er = torch.from_numpy(synth.normal(3000, 2)).cuda()
op = os.environ.get("OP", "gin")
f = {"gin": lambda: g.gin(X, 0.1, F=130), "gcn": lambda: g.gcn(X, "both", F=130),
     "gat": lambda: g.gat(X, el, er, 0.2, F=130)}[op]
for path in sys.argv[1:] or ["reg", "async"]:
    os.environ["TLP_GATHER"] = path
    g.set_schedule("dynamic")
    ref = f().clone()
    g.set_schedule("clc", 8, 1)
    y = f()
    torch.cuda.synchronize()
    print(path, "clc ok, bitwise", bool(torch.equal(y, ref)), flush=True)

"""Probe: per-launch device time of each op back-to-back vs isolated (sleep between)."""
import os, subprocess, sys, time
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch
import paper_conf_hpdc_fujh22_b200 as tlp
import synth

w = sys.argv[1] if len(sys.argv) > 1 else "reddit"
cfg = synth.CONFIGS[w]
rp, ci = synth.dataset_graph(w, device="cuda")
n, F, ld = cfg["n"], cfg["F"], cfg["ld"]
g = tlp.Graph(torch.from_numpy(rp).cuda(), torch.from_numpy(ci).cuda())
X = torch.from_numpy(synth.dataset_features(w, n)).cuda()
el = torch.from_numpy(synth.normal(n, 1)).cuda(); er = torch.from_numpy(synth.normal(n, 2)).cuda()
Y = torch.empty((n, ld), device="cuda")
ops = {"gcn": lambda: g.gcn(X, "both", Y=Y, F=F), "gin": lambda: g.gin(X, 0.1, Y=Y, F=F),
       "gat": lambda: g.gat(X, el, er, 0.2, Y=Y, F=F)}
def t1(f):
    a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    a.record(); f(); b.record(); b.synchronize(); return a.elapsed_time(b)
for k, f in ops.items():
    f(); torch.cuda.synchronize()
def smi():
    return subprocess.run(["nvidia-smi", "--query-gpu=clocks.sm,clocks.mem,power.draw,temperature.gpu,clocks_event_reasons.active", "--format=csv,noheader"], capture_output=True, text=True).stdout.strip()
print("idle:", smi())
for k, f in ops.items():
    iso = []
    for _ in range(3):
        time.sleep(1.0); iso.append(t1(f))
    b2b = [t1(f) for _ in range(6)]
    print(k, "isolated", [round(x, 2) for x in iso], "back-to-back", [round(x, 2) for x in b2b], smi())
# long back-to-back run
ts = [t1(ops["gcn"]) for _ in range(30)]
print("gcn x30 b2b", [round(x, 1) for x in ts], smi())

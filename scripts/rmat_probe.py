"""One aggregation of a pre-registered workload graph (default R-MAT-24
GCN(BOTH); `reddit gin` etc.) under scheduling / gather knobs (CUDA events,
median of N reps after warm-up).  Kernel experiment, not a bench line.
usage: python scripts/rmat_probe.py [reps] [workload] [op]"""
import os, sys, statistics
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import paper_conf_hpdc_fujh22_b200 as tlp
import synth

reps = int(sys.argv[1]) if len(sys.argv) > 1 else 8
name = sys.argv[2] if len(sys.argv) > 2 else "rmat24"
op = sys.argv[3] if len(sys.argv) > 3 else "gcn"
cfg = synth.CONFIGS[name]
rp, ci = synth.dataset_graph(name, device="cuda")
rp = torch.as_tensor(rp).cuda()
ci = torch.as_tensor(ci).cuda()
n = rp.numel() - 1
F, ld = cfg["F"], cfg["ld"]
X = torch.randn((n, ld), device="cuda")
Y = torch.empty((n, ld), device="cuda")
el = torch.randn(n, device="cuda")
er = torch.randn(n, device="cuda")


def call(g, out=None):
    if op == "gin":
        return g.gin(X, 0.1, Y=out, F=F)
    if op == "gat":
        return g.gat(X, el, er, 0.2, Y=out, F=F)
    return g.gcn(X, "both", Y=out, F=F)


def timeit(f):
    for _ in range(3):
        f()
    ts = []
    for _ in range(reps):
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        a.record(); f(); b.record(); torch.cuda.synchronize()
        ts.append(a.elapsed_time(b))
    return round(statistics.median(ts), 3)


def run(tag, g, env=None, sched=None):
    env = env or {}
    old = {k: os.environ.get(k) for k in env}
    os.environ.update(env)
    if sched:
        tlp.tlp_graph_set_schedule(g.handle, **sched)
    try:
        print(tag, timeit(lambda: call(g, Y)), flush=True)
    finally:
        for k, v in old.items():
            if v is None:
                os.environ.pop(k, None)
            else:
                os.environ[k] = v
        if sched:
            tlp.tlp_graph_set_schedule(g.handle)


g = tlp.Graph(rp, ci)
print("info", {k: g.info[k] for k in ("n_units", "n_tasks", "n_hubs", "unit_edges")}, flush=True)
ref = call(g).clone()
run("default", g)
for h in ("0", "0.25", "0.75"):
    run("TLP_HOT=" + h, g, {"TLP_HOT": h})
run("TLP_HOT_COLD=0", g, {"TLP_HOT_COLD": "0"})
run("TLP_GATHER=reg", g, {"TLP_GATHER": "reg"})
run("TLP_GATHER=async", g, {"TLP_GATHER": "async"})
run("TLP_CTAS=3", g, {"TLP_CTAS": "3"})
run("TLP_CTAS=2", g, {"TLP_CTAS": "2"})
for st in (1, 2, 8, 32):
    run(f"step={st}", g, sched=dict(step=st))
for w in (4, 16):
    run(f"wpc={w}", g, sched=dict(warps_per_cta=w))
run("TLP_BOTH=prescale", g, {"TLP_BOTH": "prescale"})
del g
torch.cuda.empty_cache()
for ue in (16, 32, 64, 256):
    g = tlp.Graph(rp, ci, opts=dict(unit_edges=ue))
    Yv = call(g)
    same = bool(torch.equal(Yv[:, :F], ref[:, :F]))
    run(f"unit_edges={ue} (bitwise same {same})", g)
    del g, Yv
    torch.cuda.empty_cache()

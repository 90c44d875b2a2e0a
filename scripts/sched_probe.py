"""Scheduler comparison: one aggregation of a workload graph
under each work scheduler -- the dynamic atomic counter (default), static,
hardware (one warp per task) and Cluster Launch Control work stealing -- with
a bitwise check against the default.  CUDA events, median of N reps.
usage: python scripts/sched_probe.py [reps] [workload:op ...]"""
import os, sys, statistics
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import paper_conf_hpdc_fujh22_b200 as tlp
import synth

reps = int(sys.argv[1]) if len(sys.argv) > 1 else 10
jobs = sys.argv[2:] or ["reddit:gin", "reddit:gat", "products:gat", "rmat24:gcn", "pubmed:gat"]


def timeit(f):
    for _ in range(3):
        f()
    ts = []
    for _ in range(reps):
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        a.record(); f(); b.record(); torch.cuda.synchronize()
        ts.append(a.elapsed_time(b))
    return round(statistics.median(ts), 4)


for job in jobs:
    name, op = job.split(":")
    cfg = synth.CONFIGS[name]
    rp, ci = synth.dataset_graph(name, device="cuda")
    rp, ci = torch.as_tensor(rp).cuda(), torch.as_tensor(ci).cuda()
    n = rp.numel() - 1
    F, ld = cfg["F"], cfg["ld"]
    gen = torch.Generator(device="cuda").manual_seed(1)
    X = torch.randn((n, ld), device="cuda", generator=gen)
    el, er = torch.randn(n, device="cuda", generator=gen), torch.randn(n, device="cuda", generator=gen)
    Y = torch.empty((n, ld), device="cuda")
    g = tlp.Graph(rp, ci)
    f = {"gcn": lambda: g.gcn(X, "both", Y=Y, F=F), "gin": lambda: g.gin(X, 0.1, Y=Y, F=F),
         "gat": lambda: g.gat(X, el, er, 0.2, Y=Y, F=F)}[op]
    f()
    ref = Y[:, :F].clone()
    order = (("dynamic", 0), ("static", 0), ("hardware", 0), ("clc", 0), ("clc", 1), ("clc", 4))
    if os.environ.get("SCHED_ORDER"):  # e.g. "clc:0,dynamic:0"
        order = [(x.split(":")[0], int(x.split(":")[1])) for x in os.environ["SCHED_ORDER"].split(",")]
    for sched, step in order:
        g.set_schedule(sched, 0, step)
        t = timeit(f)
        same = bool(torch.equal(Y[:, :F], ref))
        print(f"{name} {op} sched={sched} step={step or 'auto'}: {t} ms (bitwise same {same})", flush=True)
    g.close()
    del X, Y, rp, ci
    torch.cuda.empty_cache()

"""R-MAT-24: row-streamed cp.async units (default) vs per-row ring drains
(TLP_STREAM=0): time (CUDA events, median) and bitwise equality.

The row-streamed variant (do_unit_stream, selected by TLP_STREAM) was measured
slower and reverted (DESIGN.md R-MAT note, profiles/r01_rmat_stream_probe.log);
with the current library both modes run the same kernel."""
import os, sys, statistics
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import paper_conf_hpdc_fujh22_b200 as tlp
import synth

reps = int(sys.argv[1]) if len(sys.argv) > 1 else 8
cfg = synth.CONFIGS["rmat24"]
rp, ci = synth.dataset_graph("rmat24", device="cuda")
rp = torch.as_tensor(rp).cuda()
ci = torch.as_tensor(ci).cuda()
n = rp.numel() - 1
F, ld = cfg["F"], cfg["ld"]
X = torch.randn((n, ld), device="cuda")
g = tlp.Graph(rp, ci)


def timeit(f):
    for _ in range(3):
        f()
    ts = []
    for _ in range(reps):
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        a.record(); f(); b.record(); torch.cuda.synchronize()
        ts.append(a.elapsed_time(b))
    return round(statistics.median(ts), 3)


ops = {"gcn_both": lambda Y: g.gcn(X, "both", Y=Y, F=F), "gcn_none": lambda Y: g.gcn(X, "none", Y=Y, F=F),
       "gin": lambda Y: g.gin(X, 0.1, Y=Y, F=F), "sage": lambda Y: g.sage(X, True, Y=Y, F=F)}
for name, f in ops.items():
    res = {}
    for mode in ("0", "1", "0", "1"):
        os.environ["TLP_STREAM"] = mode
        Y = torch.full((n, ld), float("nan"), device="cuda")
        f(Y)
        torch.cuda.synchronize()
        if mode in res:
            same = bool(torch.equal(Y[:, :F], res[mode]))
        else:
            res[mode] = Y[:, :F].clone()
            same = True
        print(name, "TLP_STREAM=" + mode, timeit(lambda: f(Y)), "repeat-equal", same, flush=True)
    print(name, "bitwise stream==drain", bool(torch.equal(res["0"], res["1"])), flush=True)
    del res

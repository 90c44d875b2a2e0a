"""Small-graph latency probe (Cora GCN-BOTH, Pubmed GAT): per-call device time
(CUDA events around a captured CUDA graph of 20 calls, and plain launches) for
several unit sizes K and knobs.  usage: python scripts/small_probe.py"""
import os, sys, statistics
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import paper_conf_hpdc_fujh22_b200 as tlp
import synth


def timed(f, reps=200):
    for _ in range(20):
        f()
    torch.cuda.synchronize()
    a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    a.record()
    for _ in range(reps):
        f()
    b.record()
    torch.cuda.synchronize()
    plain = a.elapsed_time(b) / reps * 1e3
    s = torch.cuda.Stream()
    s.wait_stream(torch.cuda.current_stream())
    cg = torch.cuda.CUDAGraph()
    with torch.cuda.stream(s):
        with torch.cuda.graph(cg, stream=s):
            for _ in range(20):
                f()
    torch.cuda.current_stream().wait_stream(s)
    cg.replay()
    torch.cuda.synchronize()
    ts = []
    for _ in range(20):
        a.record(); cg.replay(); b.record(); torch.cuda.synchronize()
        ts.append(a.elapsed_time(b) / 20 * 1e3)
    return round(plain, 1), round(statistics.median(ts), 1)


if __name__ != "__main__":
    pass
else:
  for name in ("cora", "pubmed"):
      cfg = synth.CONFIGS[name]
      rp, ci = synth.dataset_graph(name, device="cuda")
      n, F, ld = cfg["n"], cfg["F"], cfg["ld"]
      X = torch.from_numpy(synth.dataset_features(name, n)).cuda()
      el = torch.from_numpy(synth.normal(n, 1)).cuda()
      er = torch.from_numpy(synth.normal(n, 2)).cuda()
      Y = torch.empty((n, ld), device="cuda")
      envs = [{}, {"TLP_BOTH": "edge"}, {"TLP_PANEL": "0"}, {"TLP_GAT": "alpha"}]
      for K in (0, 4, 8, 16, 32):
          g = tlp.Graph(torch.from_numpy(rp).cuda(), torch.from_numpy(ci).cuda(),
                        opts=dict(unit_edges=K) if K else None)
          for env in envs:
              if name == "cora" and "TLP_GAT" in env:
                  continue
              if name == "pubmed" and "TLP_BOTH" in env:
                  continue
              old = {k: os.environ.get(k) for k in env}
              os.environ.update(env)
              f = (lambda: g.gcn(X, "both", Y=Y, F=F)) if name == "cora" else (lambda: g.gat(X, el, er, 0.2, Y=Y, F=F))
              p, c = timed(f)
              print(name, "K", K or "default", env, "units", g.info["n_units"], "us plain", p, "graph", c, flush=True)
              for k, v in old.items():
                  if v is None:
                      os.environ.pop(k, None)
                  else:
                      os.environ[k] = v
          g.close()

"""Graph-create timing probe: creates the Reddit-shaped graph several times
(the first call includes lazy module loading) and prints create_ms."""
import sys, os, time
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import paper_conf_hpdc_fujh22_b200 as tlp
import synth
name = sys.argv[1] if len(sys.argv) > 1 else "reddit"
rp, ci = synth.dataset_graph(name, device="cuda")
rpd = torch.as_tensor(rp).cuda() if not torch.is_tensor(rp) else rp.cuda()
cid = torch.as_tensor(ci).cuda() if not torch.is_tensor(ci) else ci.cuda()
n = rpd.numel() - 1
for i in range(4):
    torch.cuda.synchronize()
    t = time.perf_counter()
    g = tlp.Graph(rpd, cid, n_src=n)
    torch.cuda.synchronize()
    print(name, "create", i, "wall %.2f ms" % (1e3 * (time.perf_counter() - t)), "create_ms", g.info["create_ms"])
    g.close()

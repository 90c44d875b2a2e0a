"""Rank body of tests/test_dist_torchrun.py (launched by torch.distributed.run,
one rank per GPU).  Every rank builds the dist handle of the same seeded graph,
runs each dist aggregation both ways -- aggregate + grouped-broadcast
all-gather, and the fused peer-store kernel (NEXT-2) into a symmetric buffer --
and checks Y_full bit for bit against the single-GPU result computed on the
same rank, plus sampled rows against the fp64 oracle (so the multi-destination
output is held to the oracle, not only to itself).  Exits non-zero on any
mismatch; rank 0 prints one JSON line."""
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import numpy as np  # noqa: E402
import torch  # noqa: E402
import torch.distributed as dist  # noqa: E402

import oracle  # noqa: E402
import paper_conf_hpdc_fujh22_b200 as tlp  # noqa: E402
import synth  # noqa: E402


def main():
    rank = int(os.environ["RANK"])
    world = int(os.environ["WORLD_SIZE"])
    local = int(os.environ.get("LOCAL_RANK", "0"))
    torch.cuda.set_device(local)
    dev = torch.device("cuda", local)
    dist.init_process_group("nccl", device_id=dev, rank=rank, world_size=world)
    n = 6000
    rp, ci = synth.chung_lu(n, 240000, 0.45, 61, device="cpu")
    F, ld = 130, 132
    Xh = synth.features(n, F, ld, seed=7)
    elh, erh = synth.normal(n, 8), synth.normal(n, 9)
    X = torch.from_numpy(Xh).to(dev)
    el, er = torch.from_numpy(elh).to(dev), torch.from_numpy(erh).to(dev)
    opts = dict(hub_threshold=128, hub_chunk=64)
    comm = tlp.comm_from_torch()
    h = tlp.tlp_dist_graph_create(comm, torch.from_numpy(rp).to(dev), torch.from_numpy(ci).to(dev), opts=opts)
    g1 = tlp.Graph(torch.from_numpy(rp).to(dev), torch.from_numpy(ci).to(dev), opts=opts)
    b = tlp.tlp_dist_bounds(h, world)
    assert np.array_equal(b, oracle.partition(rp, world)), "partition bounds"
    ops = {
        "gcn": (dict(norm="both"), lambda: g1.gcn(X, "both", F=F),
                lambda rows: oracle.gcn(rp, ci, Xh, "both", rows=rows, F=F)),
        "gin": (dict(eps=0.1), lambda: g1.gin(X, 0.1, F=F),
                lambda rows: oracle.gin(rp, ci, Xh, 0.1, rows=rows, F=F)),
        "gat": (dict(el=el, er=er, slope=0.2), lambda: g1.gat(X, el, er, 0.2, F=F),
                lambda rows: oracle.gat(rp, ci, Xh, elh, erh, 0.2, rows=rows, F=F)),
        "sage": (dict(include_self=True), lambda: g1.sage(X, True, F=F),
                 lambda rows: oracle.sage(rp, ci, Xh, include_self=True, rows=rows, F=F)),
    }
    rng = np.random.default_rng(5)
    rows = np.unique(np.concatenate([rng.choice(n, 300, replace=False), b[:-1].clip(max=n - 1)]))
    report = {}
    # the symmetric buffer: NCCL window (default) or CUDA IPC (TLP_SYM=ipc)
    Ysym, ptr = tlp.tlp_comm_alloc_symmetric(comm, n, ld)
    sym_kind = tlp.tlp_comm_symmetric_kind(comm, ptr)
    for op, (kw, single, ref) in ops.items():
        Y1 = single()
        torch.cuda.synchronize()
        # (a) aggregate + grouped-broadcast all-gather
        Yf = torch.full((n, ld), float("nan"), device=dev)
        tlp.tlp_dist_aggregate(h, comm, op, X, Yf, F=F, **kw)
        tlp.tlp_comm_wait(comm, torch.cuda.current_stream(dev), 120.0)
        assert torch.equal(Yf[:, :F], Y1), f"{op}: dist all-gather != single GPU"
        # (b) fused: one kernel stores every row into Y_full on every rank
        Ysym.fill_(float("nan"))
        tlp.tlp_dist_aggregate_fused(h, comm, op, X, Ysym, F=F, **kw)
        tlp.tlp_comm_wait(comm, torch.cuda.current_stream(dev), 120.0)
        assert torch.equal(Ysym[:, :F], Y1), f"{op}: fused != single GPU"
        assert torch.isnan(Ysym[:, F:]).all(), f"{op}: fused wrote pad columns"
        Yr, Ar = ref(rows)
        ok, worst = oracle.within_tolerance(Ysym[torch.from_numpy(rows).to(dev), :F].cpu().numpy(), Yr, Ar)
        assert ok, f"{op}: fused output vs oracle worst err/tol {worst:.3g}"
        report[op] = round(worst, 4)
    assert tlp.tlp_comm_async_error(comm) == 0
    tlp.tlp_comm_free_symmetric(comm, ptr)
    tlp.tlp_graph_destroy(h)
    g1.close()
    tlp.tlp_comm_destroy(comm)
    dist.destroy_process_group()
    if rank == 0:
        print(json.dumps({"world": world, "worst_err_over_tol": report, "bounds": b.tolist(),
                          "symmetric_buffer": sym_kind}))


if __name__ == "__main__":
    main()

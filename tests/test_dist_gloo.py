"""World-size-2 gloo test of the N>1 host logic (runs on CPU): edge-balanced
row partition from the library, per-rank row slices with global sources and a
row offset, and the all-gather of row slabs as P in-place broadcasts (the
grouped ncclBroadcast of tlp_dist_allgather_rows).  The per-rank local compute
is the oracle here (no GPU); the assembled Y_full must be bitwise equal to the
single-process oracle result, as the dist contract promises for the GPU path."""
import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, world, port, q):
    try:
        os.environ["MASTER_ADDR"] = "127.0.0.1"
        os.environ["MASTER_PORT"] = str(port)
        dist.init_process_group("gloo", rank=rank, world_size=world)
        import oracle
        import synth
        import paper_conf_hpdc_fujh22_b200 as tlp
        n = 300
        rp, ci = synth.chung_lu(n, 4000, 0.6, 9, device="cpu")
        F = 5
        X = synth.features(n, F, 8, seed=1)
        el, er = synth.normal(n, 2), synth.normal(n, 3)
        b = tlp.tlp_partition_rows(rp, world)
        # every rank derives the same bounds
        allb = [None] * world
        dist.all_gather_object(allb, b.tolist())
        assert all(x == allb[0] for x in allb)
        r0, r1 = int(b[rank]), int(b[rank + 1])
        sl_rp = rp[r0:r1 + 1] - rp[r0]
        sl_ci = ci[rp[r0]:rp[r1]]
        outs = {}
        for op in ("gcn", "gin", "gat"):
            Y = torch.zeros((n, F), dtype=torch.float64)
            if r1 > r0:
                if op == "gcn":
                    # BOTH needs the GLOBAL out-degree: evaluate the slice rows on the full CSR
                    loc, _ = oracle.gcn(rp, ci, X, "both", rows=np.arange(r0, r1), F=F)
                elif op == "gin":
                    loc, _ = oracle.gin(sl_rp, sl_ci, X, 0.1, row_offset=r0, F=F)
                else:
                    loc, _ = oracle.gat(sl_rp, sl_ci, X, el, er, 0.2, row_offset=r0, F=F)
                Y[r0:r1] = torch.from_numpy(loc)
            for r in range(world):  # grouped in-place broadcast of each slab
                a, c = int(b[r]), int(b[r + 1])
                if c > a:
                    slab = Y[a:c].contiguous()
                    dist.broadcast(slab, src=r)
                    Y[a:c] = slab
            outs[op] = Y.numpy()
        ref = {"gcn": oracle.gcn(rp, ci, X, "both", F=F)[0],
               "gin": oracle.gin(rp, ci, X, 0.1, F=F)[0],
               "gat": oracle.gat(rp, ci, X, el, er, 0.2, F=F)[0]}
        for op in outs:
            assert np.array_equal(outs[op], ref[op]), op
        dist.destroy_process_group()
        q.put((rank, "ok"))
    except Exception as e:  # pragma: no cover - reported to the parent
        import traceback
        q.put((rank, traceback.format_exc()))


@pytest.mark.parametrize("world", [2])
def test_dist_host_logic_gloo(world):
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    ps = [ctx.Process(target=_worker, args=(r, world, port, q)) for r in range(world)]
    for p in ps:
        p.start()
    res = [q.get(timeout=300) for _ in ps]
    for p in ps:
        p.join(timeout=60)
    for rank, msg in res:
        assert msg == "ok", f"rank {rank}: {msg}"

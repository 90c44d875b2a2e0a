"""All-row parity at config scale: the
unchanged fp64 oracle driven over disjoint chunks of destination rows in a pool
of processes (one per host core).  Rows are independent, so every oracle
value is the single-threaded one, bit for bit.  The inputs and the GPU output
are written once to a tmpfs directory and memory-mapped by the workers; each
worker compares its rows element by element with the north-star criterion
|err| <= 1e-5 * sum|terms| + 1e-6 and returns only (rows, worst ratio, bad
elements), so no large array crosses a pipe.

Test infrastructure: imported by tests/ only."""
from __future__ import annotations

import multiprocessing as mp
import os
import shutil
import tempfile

import numpy as np


def _load(d, name):
    p = os.path.join(d, name + ".npy")
    return np.load(p, mmap_mode="r") if os.path.exists(p) else None


def _task(job):
    import oracle
    d, op, params, rows = job
    rp = np.asarray(_load(d, "rp"))
    ci = _load(d, "ci")
    X = _load(d, "X")
    Yg = _load(d, "Y")
    F = params["F"]
    if op == "gcn":
        Yr, Ar = oracle.gcn(rp, ci, X, params["norm"], rows=rows, F=F, n_src=X.shape[0])
    elif op == "gin":
        Yr, Ar = oracle.gin(rp, ci, X, params["eps"], rows=rows, F=F)
    elif op == "sage":
        Yr, Ar = oracle.sage(rp, ci, X, include_self=params["include_self"], rows=rows, F=F)
    elif op == "gat":
        Yr, Ar = oracle.gat(rp, ci, X, _load(d, "el"), _load(d, "er"), params["slope"], rows=rows, F=F)
    elif op == "gat_mh":
        H = params["heads"]
        Yr, Ar = oracle.gat_mh(rp, ci, X, np.asarray(_load(d, "el")).reshape(-1, H),
                               np.asarray(_load(d, "er")).reshape(-1, H), H, params["slope"],
                               rows=rows, Fh=F // H)
    else:
        raise ValueError(op)
    Yt = np.asarray(Yg[rows, :F], dtype=np.float64)
    err = np.abs(Yt - Yr)
    tol = 1e-5 * Ar + 1e-6
    bad = int(np.count_nonzero(~(err <= tol)))  # NaN counts as bad
    worst = float(np.nanmax(err / tol)) if err.size else 0.0
    return len(rows), worst, bad


def check_rows(op, rp, ci, X, Y_gpu, rows=None, procs=None, chunk=None, el=None, er=None, **params):
    """Compare the GPU output Y_gpu (numpy fp32 [n_dst, >= F]) with the oracle on
    `rows` (all rows by default).  params: F and the op's scalars (norm, eps,
    slope, include_self, heads).  Returns dict(rows, worst, bad)."""
    n_dst = len(rp) - 1
    rows = np.arange(n_dst, dtype=np.int64) if rows is None else np.asarray(rows, dtype=np.int64)
    procs = procs or max(1, len(os.sched_getaffinity(0)))
    if chunk is None:
        # ~ equal edge counts per task, a few tasks per process
        chunk = max(64, min(4096, len(rows) // (procs * 8) + 1))
    base = "/dev/shm" if os.path.isdir("/dev/shm") else None
    d = tempfile.mkdtemp(prefix="tlp_parity_", dir=base)
    try:
        arrays = {"rp": rp, "ci": ci, "X": X, "Y": Y_gpu, "el": el, "er": er}
        for k, v in arrays.items():
            if v is not None:
                np.save(os.path.join(d, k + ".npy"), np.ascontiguousarray(v))
        jobs = [(d, op, params, rows[i:i + chunk]) for i in range(0, len(rows), chunk)]
        with mp.get_context("spawn").Pool(min(procs, len(jobs))) as pool:
            res = pool.map(_task, jobs, chunksize=1)
    finally:
        shutil.rmtree(d, ignore_errors=True)
    return {"rows": int(sum(r[0] for r in res)), "worst": max(r[1] for r in res),
            "bad": int(sum(r[2] for r in res))}

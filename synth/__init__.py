"""Seeded synthetic inputs for the TLPGNN aggregation hot path.

This module is shared by the oracle side (tests) and the CUDA side (tests,
bench) and therefore holds NONE of the method's arithmetic: it only draws
graphs and feature values.  It imports neither ``oracle`` nor the product
package.  The recipe is pre-registered in DESIGN.md "Input recipe" (SURVEY
8(d) d1) and must not be tuned to the kernel.

* ``chung_lu``: generator G1 ("dataset-shaped", Cora/Pubmed/Reddit/products):
  undirected Chung-Lu with rank weights w_i = (i+1)^-alpha; exactly M = E/2
  distinct non-loop unordered pairs accepted in draw order; both directions
  emitted (exactly E directed edges, symmetric, no self-loops, no multi-edges);
  a seeded random relabelling; in-edge CSR sorted by (dst, src).
* ``rmat``: generator G2 (Graph500 R-MAT, a,b,c,d = .57,.19,.19,.05).
* ``features``: X ~ U[-1,1) fp32 (the paper: "random 32-bits floating
  numbers"), stress variant U[0,1); ``normal`` for el/er.

Random numbers come from numpy's PCG64 (chung_lu, features) or a counter-based
splitmix64 hash (rmat, so the 2^28-pair graph can be drawn on the GPU); the
structural steps (dedupe, sort, CSR build) are deterministic torch ops that
give identical results on CPU and CUDA.
"""
from __future__ import annotations

import math
import os

import numpy as np

# Pre-registered configs (BASELINE.json "configs").
CONFIGS = {
    "cora": dict(n=2708, e=10556, F=1433, ld=1436, alpha=0.58, seed=1, op="gcn"),
    "pubmed": dict(n=19717, e=88648, F=500, ld=500, alpha=0.42, seed=2, op="gat"),
    "reddit": dict(n=232965, e=114615892, F=602, ld=604, alpha=0.34, seed=3, op="gcn+gin"),
    "products": dict(n=2449029, e=123718280, F=100, ld=100, alpha=0.44, seed=4, op="gat"),
    "rmat24": dict(scale=24, edge_factor=16, F=128, ld=128, seed=5, op="gcn2"),
}
FEATURE_SEED_BASE = 100  # feature seed = 100 + config index
CONFIG_INDEX = {"cora": 1, "pubmed": 2, "reddit": 3, "products": 4, "rmat24": 5}
SLOPE = 0.2   # GAT LeakyReLU slope (c2 #6)
EPS = 0.1     # GIN eps used by configs and tests (c2 #9)


def _torch():
    import torch
    return torch


def _device(device):
    torch = _torch()
    if device is None:
        device = "cuda" if torch.cuda.is_available() else "cpu"
    return torch.device(device)


def _first_distinct(keys):
    """Ascending positions of the first occurrence of every distinct value."""
    torch = _torch()
    perm = torch.argsort(keys, stable=True)
    sk = keys[perm]
    first = torch.ones_like(sk, dtype=torch.bool)
    first[1:] = sk[1:] != sk[:-1]
    pos, _ = torch.sort(perm[first])
    return pos


def _csr_from_pairs(a, b, n, perm):
    """Symmetrise unordered pairs (a,b), relabel with perm, build the in-edge
    CSR sorted by (dst, src).  Returns numpy (rowptr int64, colidx int32)."""
    torch = _torch()
    src = torch.cat([a, b])
    dst = torch.cat([b, a])
    del a, b
    src = perm[src]
    dst = perm[dst]
    key = dst * n + src
    del src
    key, _ = torch.sort(key)
    dst = key // n
    col = (key - dst * n).to(torch.int32)
    del key
    counts = torch.bincount(dst, minlength=n)
    del dst
    rowptr = torch.zeros(n + 1, dtype=torch.int64, device=counts.device)
    rowptr[1:] = torch.cumsum(counts, 0)
    return rowptr.cpu().numpy(), col.cpu().numpy()


def chung_lu(n, e, alpha, seed, device=None):
    """Generator G1.  Returns (rowptr int64[n+1], colidx int32[e]) numpy arrays."""
    torch = _torch()
    assert e % 2 == 0, "symmetric graph needs an even edge count"
    m = e // 2
    dev = _device(device)
    rng = np.random.Generator(np.random.PCG64(seed))
    w = (np.arange(n, dtype=np.float64) + 1.0) ** (-float(alpha))
    cdf = np.cumsum(w)
    cdf /= cdf[-1]
    cdf_t = torch.from_numpy(cdf).to(dev)
    keys = torch.empty(0, dtype=torch.int64, device=dev)
    have = 0
    while True:
        need = m - have
        batch = int(need * 1.15) + 1024
        r = torch.from_numpy(rng.random((batch, 2))).to(dev)
        u = torch.searchsorted(cdf_t, r[:, 0].contiguous(), right=True).clamp_(max=n - 1)
        v = torch.searchsorted(cdf_t, r[:, 1].contiguous(), right=True).clamp_(max=n - 1)
        del r
        keep = u != v
        lo = torch.minimum(u, v)[keep]
        hi = torch.maximum(u, v)[keep]
        keys = torch.cat([keys, lo * n + hi])
        del u, v, lo, hi, keep
        # keep the distinct values in order of first draw (acceptance order)
        keys = keys[_first_distinct(keys)]
        have = keys.numel()
        if have >= m:
            break
    keys = keys[:m]
    a = keys // n
    b = keys - a * n
    del keys
    perm = torch.from_numpy(rng.permutation(n)).to(dev)
    return _csr_from_pairs(a, b, n, perm)


# ---- counter-based RNG for R-MAT (splitmix64 finaliser) -------------------
_M1 = 0xBF58476D1CE4E5B9
_M2 = 0x94D049BB133111EB
_GOLD = 0x9E3779B97F4A7C15


def _to_signed(x):
    return x - (1 << 64) if x >= (1 << 63) else x


def _splitmix(ctr):
    """splitmix64 on an int64 tensor (two's complement wraparound)."""
    torch = _torch()
    z = ctr * _to_signed(_GOLD)
    z = (z ^ ((z >> 30) & ((1 << 34) - 1))) * _to_signed(_M1)
    z = (z ^ ((z >> 27) & ((1 << 37) - 1))) * _to_signed(_M2)
    z = z ^ ((z >> 31) & ((1 << 33) - 1))
    return z


def _uniform01(ctr):
    """53-bit uniform in [0,1) from a counter tensor."""
    torch = _torch()
    z = _splitmix(ctr)
    return ((z >> 11) & ((1 << 53) - 1)).to(torch.float64) * (1.0 / (1 << 53))


def rmat(scale, edge_factor, seed, a=0.57, b=0.19, c=0.19, device=None):
    """Generator G2 (Graph500 R-MAT, no noise): M = edge_factor * 2^scale distinct
    non-loop unordered pairs accepted in draw order, symmetrised (E = 2M),
    seeded relabel.  Returns numpy (rowptr, colidx)."""
    torch = _torch()
    n = 1 << scale
    m = edge_factor * n
    dev = _device(device)
    keys = torch.empty(0, dtype=torch.int64, device=dev)
    drawn = 0
    have = 0
    while True:
        need = m - have
        batch = int(need * 1.25) + 1024
        idx = torch.arange(drawn, drawn + batch, dtype=torch.int64, device=dev)
        drawn += batch
        u = torch.zeros(batch, dtype=torch.int64, device=dev)
        v = torch.zeros(batch, dtype=torch.int64, device=dev)
        base = (idx * (scale + 1) + (seed << 40))
        for lvl in range(scale):
            r = _uniform01(base + lvl)
            bit_u = (r >= a + b).to(torch.int64)              # quadrants c, d
            bit_v = ((r >= a) & (r < a + b)) | (r >= a + b + c)  # quadrants b, d
            u = (u << 1) | bit_u
            v = (v << 1) | bit_v.to(torch.int64)
            del r, bit_u, bit_v
        del base, idx
        keep = u != v
        lo = torch.minimum(u, v)[keep]
        hi = torch.maximum(u, v)[keep]
        del u, v, keep
        keys = torch.cat([keys, lo * n + hi])
        del lo, hi
        keys = keys[_first_distinct(keys)]
        have = keys.numel()
        if have >= m:
            break
    keys = keys[:m]
    a_ = keys // n
    b_ = keys - a_ * n
    del keys
    g = torch.Generator(device="cpu")
    g.manual_seed(seed)
    perm = torch.randperm(n, generator=g).to(dev)
    return _csr_from_pairs(a_, b_, n, perm)


# ---- feature values -------------------------------------------------------

def features(n, F, ld=None, seed=0, low=-1.0, high=1.0):
    """X ~ U[low, high) fp32 of shape [n, ld]; pad columns [F, ld) are 0."""
    ld = F if ld is None else ld
    rng = np.random.Generator(np.random.PCG64(seed))
    X = np.zeros((n, ld), np.float32)
    if n and F:
        X[:, :F] = rng.random((n, F), dtype=np.float32) * np.float32(high - low) + np.float32(low)
    return X


def normal(n, seed):
    rng = np.random.Generator(np.random.PCG64(seed))
    return rng.standard_normal(n, dtype=np.float32)


def edge_weights(e, seed):
    """U(0,1] fp32 edge weights (weighted test variants only)."""
    rng = np.random.Generator(np.random.PCG64(seed))
    return (np.float32(1.0) - rng.random(e, dtype=np.float32)).astype(np.float32)


# ---- small structured graphs for edge cases --------------------------------

def csr_from_edges(n_dst, src, dst):
    """In-edge CSR of the directed edges src->dst, CSR order = stable by dst,
    keeping the given order of edges within a row (multi-edges kept)."""
    src = np.asarray(src, np.int64)
    dst = np.asarray(dst, np.int64)
    order = np.argsort(dst, kind="stable")
    colidx = src[order].astype(np.int32)
    counts = np.bincount(dst, minlength=n_dst) if dst.size else np.zeros(n_dst, np.int64)
    rowptr = np.zeros(n_dst + 1, np.int64)
    rowptr[1:] = np.cumsum(counts)
    return rowptr, colidx


def figure1_star(self_loops=True):
    """The Figure-1 graph as read in c2 #15: undirected star A-B, A-C, A-D
    (A=0..D=3), plus self-loops on all four when self_loops."""
    src = [1, 2, 3, 0, 0, 0]
    dst = [0, 0, 0, 1, 2, 3]
    if self_loops:
        src += [0, 1, 2, 3]
        dst += [0, 1, 2, 3]
    rowptr, colidx = csr_from_edges(4, src, dst)
    # sort each row by source id (CSR order (dst, src))
    for v in range(4):
        colidx[rowptr[v]:rowptr[v + 1]].sort()
    return rowptr, colidx


def random_graph(n_dst, n_src, e, seed, self_loops=True, multi=True, isolated_tail=0):
    """Random directed multigraph with uniform endpoints (edge-case tests).
    The last `isolated_tail` destinations get no in-edges."""
    rng = np.random.Generator(np.random.PCG64(seed))
    nd = max(n_dst - isolated_tail, 0)
    if nd == 0 or n_src == 0:
        return csr_from_edges(n_dst, [], [])
    src = rng.integers(0, n_src, e)
    dst = rng.integers(0, nd, e)
    if not self_loops:
        keep = src != dst
        src, dst = src[keep], dst[keep]
    if not multi:
        k = np.unique(dst * n_src + src)
        dst, src = k // n_src, k % n_src
    return csr_from_edges(n_dst, src, dst)


def power_law_rows(n, degrees, n_src, seed):
    """CSR with prescribed per-row in-degrees and uniform random sources."""
    rng = np.random.Generator(np.random.PCG64(seed))
    degrees = np.asarray(degrees, np.int64)
    rowptr = np.zeros(n + 1, np.int64)
    rowptr[1:] = np.cumsum(degrees)
    colidx = rng.integers(0, n_src, int(rowptr[-1])).astype(np.int32)
    return rowptr, colidx


def degree_stats(rowptr):
    d = np.diff(rowptr)
    if d.size == 0:
        return dict(max=0, mean=0.0, p99=0)
    return dict(max=int(d.max()), mean=float(d.mean()), p99=int(np.percentile(d, 99)))


# ---- dataset-shaped graphs with an optional on-disk cache -------------------

def _cache_dir():
    d = os.environ.get("TLP_SYNTH_CACHE")
    return d


def dataset_graph(name, device=None):
    """The pre-registered graph of config `name` (cached under $TLP_SYNTH_CACHE
    when set; nothing depends on the cache)."""
    cfg = CONFIGS[name]
    cdir = _cache_dir()
    if cdir:
        p = os.path.join(cdir, f"{name}_seed{cfg['seed']}")
        if os.path.exists(p + "_rowptr.npy") and os.path.exists(p + "_colidx.npy"):
            return np.load(p + "_rowptr.npy"), np.load(p + "_colidx.npy")
    if name == "rmat24":
        g = rmat(cfg["scale"], cfg["edge_factor"], cfg["seed"], device=device)
    else:
        g = chung_lu(cfg["n"], cfg["e"], cfg["alpha"], cfg["seed"], device=device)
    if cdir:
        os.makedirs(cdir, exist_ok=True)
        # atomic per file (several ranks may generate the same graph at once);
        # colidx lands last, and readers require both files
        for suffix, arr in (("_rowptr.npy", g[0]), ("_colidx.npy", g[1])):
            tmp = "%s%s.%d.tmp.npy" % (p, suffix, os.getpid())
            np.save(tmp, arr)
            os.replace(tmp, p + suffix)
    return g


def dataset_features(name, n):
    cfg = CONFIGS[name]
    return features(n, cfg["F"], cfg["ld"], seed=FEATURE_SEED_BASE + CONFIG_INDEX[name])

"""All-row parity at the BASELINE.json config sizes (the paper
measures exactly this operator): the CUDA path, through the C ABI,
in the launch configuration bench.py times, against the unchanged fp64 oracle on
EVERY destination row of Reddit (GCN-BOTH, GIN, GAT in both softmax modes,
GraphSage; plus the non-negative stress input of SURVEY c3 P8, the worst case
for fp32 cancellation-free error growth) and products (GAT, 4-head GAT), and on
>= 1 % random rows plus EVERY hub row of the R-MAT-24 two-layer GCN (layer 2
against the oracle applied to the GPU's fp32 layer-1 output, reading R22).
The oracle runs over row chunks in a process pool (tests/oracle_pool.py)."""
import numpy as np
import pytest

import synth
from oracle_pool import check_rows

pytestmark = pytest.mark.gpu

torch = pytest.importorskip("torch")
DEV = "cuda:0"


@pytest.fixture(scope="module")
def tlp():
    import paper_conf_hpdc_fujh22_b200 as m
    return m


def _t(a):
    return torch.from_numpy(np.ascontiguousarray(a)).to(DEV)


def _host(Y):
    torch.cuda.synchronize()
    return Y.cpu().numpy()


def _ok(name, r, n_rows):
    assert r["rows"] == n_rows, (name, r)
    assert r["bad"] == 0, f"{name}: {r['bad']} elements out of tolerance (worst err/tol {r['worst']:.3g})"
    return r["worst"]


@pytest.fixture(scope="module")
def reddit():
    return synth.dataset_graph("reddit")


@pytest.mark.parametrize("nonneg", [False, True])
def test_reddit_gcn_gin_sage_all_rows(tlp, reddit, nonneg):
    cfg = synth.CONFIGS["reddit"]
    n, F, ld = cfg["n"], cfg["F"], cfg["ld"]
    rp, ci = reddit
    Xh = synth.features(n, F, ld, seed=103, low=0.0 if nonneg else -1.0)
    X = _t(Xh)
    g = tlp.Graph(_t(rp), _t(ci))
    Y = _host(g.gcn(X, "both", F=F))
    _ok("reddit gcn", check_rows("gcn", rp, ci, Xh, Y, F=F, norm="both"), n)
    Y = _host(g.gin(X, synth.EPS, F=F))
    _ok("reddit gin", check_rows("gin", rp, ci, Xh, Y, F=F, eps=synth.EPS), n)
    if not nonneg:
        Y = _host(g.sage(X, True, F=F))
        _ok("reddit sage", check_rows("sage", rp, ci, Xh, Y, F=F, include_self=True), n)
    g.close()


@pytest.mark.parametrize("gat_mode", ["auto", "online"])
def test_reddit_gat_all_rows(tlp, reddit, monkeypatch, gat_mode):
    if gat_mode != "auto":
        monkeypatch.setenv("TLP_GAT", gat_mode)
    cfg = synth.CONFIGS["reddit"]
    n, F, ld = cfg["n"], cfg["F"], cfg["ld"]
    rp, ci = reddit
    Xh = synth.features(n, F, ld, seed=103)
    el, er = synth.normal(n, 301), synth.normal(n, 302)
    g = tlp.Graph(_t(rp), _t(ci))
    Y = _host(g.gat(_t(Xh), _t(el), _t(er), synth.SLOPE, F=F))
    _ok("reddit gat " + gat_mode, check_rows("gat", rp, ci, Xh, Y, el=el, er=er, F=F, slope=synth.SLOPE), n)
    g.close()


def test_products_gat_all_rows(tlp):
    cfg = synth.CONFIGS["products"]
    n, F = cfg["n"], cfg["F"]
    rp, ci = synth.dataset_graph("products")
    Xh = synth.dataset_features("products", n)
    el, er = synth.normal(n, 401), synth.normal(n, 402)
    g = tlp.Graph(_t(rp), _t(ci))
    Y = _host(g.gat(_t(Xh), _t(el), _t(er), synth.SLOPE, F=F))
    _ok("products gat", check_rows("gat", rp, ci, Xh, Y, el=el, er=er, F=F, slope=synth.SLOPE), n)
    H = 4
    el4, er4 = synth.normal(n * H, 403), synth.normal(n * H, 404)
    Y = _host(g.gat_mh(_t(Xh), _t(el4.reshape(n, H)), _t(er4.reshape(n, H)), H, synth.SLOPE, F=F))
    _ok("products gat4", check_rows("gat_mh", rp, ci, Xh, Y, el=el4, er=er4, F=F, heads=H,
                                    slope=synth.SLOPE), n)
    g.close()


def test_rmat24_two_layers_rows_and_all_hubs(tlp):
    cfg = synth.CONFIGS["rmat24"]
    n = 1 << cfg["scale"]
    F = cfg["F"]
    rp, ci = synth.dataset_graph("rmat24")
    Xh = synth.features(n, F, F, seed=105)
    g = tlp.Graph(_t(rp), _t(ci))
    H = g.info["hub_threshold"]
    deg = np.diff(rp)
    hubs = np.flatnonzero(deg > H)
    assert len(hubs) == g.info["n_hubs"]
    rng = np.random.default_rng(24)
    rows = np.unique(np.concatenate([hubs, rng.choice(n, n // 100, replace=False)]))
    X = _t(Xh)
    Y1 = g.gcn(X, "both")
    Y2 = g.gcn(Y1, "both")
    Y1h, Y2h = _host(Y1), _host(Y2)
    _ok("rmat layer 1", check_rows("gcn", rp, ci, Xh, Y1h, rows=rows, F=F, norm="both"), len(rows))
    _ok("rmat layer 2", check_rows("gcn", rp, ci, Y1h, Y2h, rows=rows, F=F, norm="both"), len(rows))
    g.close()

"""Pins of the fp64 oracle against things other than itself.

P1 Figure-1 star worked by hand (tests/golden/figure1_star.json)
P2 dense brute force on <=64-vertex graphs (numpy matrices, no CSR loops)
P3 scipy.sparse CSR matmul at Cora/Pubmed scale
P4 closed-form invariants, P5 softmax rows sum to one, P6 structure.

Every function in oracle/tlp_oracle.c is exercised by at least one pin chosen
so a dropped term, wrong sign/index or transposed operand fails it.
"""
import json
import math
import os

import numpy as np
import pytest

import oracle
import synth

GOLD = os.path.join(os.path.dirname(__file__), "golden", "figure1_star.json")


def _star():
    with open(GOLD) as f:
        return json.load(f)


# ---------------------------------------------------------------- P1 --------

@pytest.mark.parametrize("norm", ["none", "right", "both"])
def test_p1_star_gcn(norm):
    g = _star()
    s = g["with_self_loops"]
    rp, ci = synth.figure1_star(self_loops=True)
    assert rp.tolist() == s["rowptr"] and ci.tolist() == s["colidx"]
    X = np.array(g["x"], np.float32).reshape(-1, 1)
    Y, A = oracle.gcn(rp, ci, X, norm)
    np.testing.assert_allclose(Y.ravel(), s["gcn_" + norm], rtol=1e-15, atol=0)
    # all x > 0, so sum|terms| equals the sum itself
    np.testing.assert_allclose(A.ravel(), s["gcn_" + norm], rtol=1e-15)


def test_p1_star_degrees():
    s = _star()["with_self_loops"]
    rp, ci = synth.figure1_star(self_loops=True)
    assert oracle.in_degree(rp).tolist() == s["in_deg"]
    assert oracle.out_degree(ci, 4).tolist() == s["in_deg"]


def test_p1_star_gin():
    g = _star()
    s = g["without_self_loops"]
    rp, ci = synth.figure1_star(self_loops=False)
    assert rp.tolist() == s["rowptr"] and ci.tolist() == s["colidx"]
    X = np.array(g["x"], np.float32).reshape(-1, 1)
    Y, _ = oracle.gin(rp, ci, X, 0.5)
    np.testing.assert_allclose(Y.ravel(), s["gin_eps0.5"], rtol=1e-15)


@pytest.mark.parametrize("er_val,key", [(0.0, "gat_slope0.2_el_lnx_er0"),
                                         (-10.0, "gat_slope0.2_el_lnx_er-10")])
def test_p1_star_gat(er_val, key):
    g = _star()
    s = g["with_self_loops"]
    rp, ci = synth.figure1_star(self_loops=True)
    X = np.array(g["x"], np.float32).reshape(-1, 1)
    el = np.log(np.array(g["x"], np.float64)).astype(np.float32)
    er = np.full(4, er_val, np.float32)
    Y, A = oracle.gat(rp, ci, X, el, er, 0.2)
    # el is ln(x) rounded to fp32 (relative 6e-8), which perturbs alpha by ~1e-7
    np.testing.assert_allclose(Y.ravel(), s[key], rtol=1e-6)


def test_p1_star_gat_uniform_scores_equal_mean():
    rp, ci = synth.figure1_star(self_loops=True)
    X = np.array([1, 2, 3, 4], np.float32).reshape(-1, 1)
    Y, _ = oracle.gat(rp, ci, X, np.zeros(4, np.float32), np.zeros(4, np.float32), 0.2)
    np.testing.assert_allclose(Y.ravel(), _star()["with_self_loops"]["gcn_right"], rtol=1e-15)


# ---------------------------------------------------------------- P2 --------

def _dense_adj(rp, ci, n_dst, n_src, ew=None):
    """A[v,u] = sum of w_e over the edges u->v (multi-edges add up)."""
    A = np.zeros((n_dst, n_src))
    C = np.zeros((n_dst, n_src))
    for v in range(n_dst):
        for e in range(rp[v], rp[v + 1]):
            A[v, ci[e]] += 1.0 if ew is None else float(ew[e])
            C[v, ci[e]] += 1.0
    return A, C


def _brute_gcn(rp, ci, X, norm, n_src, ew=None):
    n_dst = len(rp) - 1
    A, C = _dense_adj(rp, ci, n_dst, n_src, ew)
    din = C.sum(1)
    dout = C.sum(0)
    if norm == "none":
        cin, cout = np.ones(n_dst), np.ones(n_src)
    elif norm == "right":
        cin, cout = 1.0 / np.maximum(din, 1), np.ones(n_src)
    else:
        cin, cout = 1.0 / np.sqrt(np.maximum(din, 1)), 1.0 / np.sqrt(np.maximum(dout, 1))
    return np.diag(cin) @ A @ np.diag(cout) @ X.astype(np.float64)


def _brute_gat(rp, ci, X, el, er, slope, n_src):
    n_dst = len(rp) - 1
    _, C = _dense_adj(rp, ci, n_dst, n_src)
    T = er.astype(np.float64)[:n_dst, None] + el.astype(np.float64)[None, :]
    S = np.where(T >= 0, T, slope * T)
    S = np.where(C > 0, S, -np.inf)
    m = S.max(1, keepdims=True)
    m = np.where(np.isfinite(m), m, 0.0)
    P = C * np.exp(S - m)
    Z = P.sum(1, keepdims=True)
    P = np.divide(P, Z, out=np.zeros_like(P), where=Z > 0)
    return P @ X.astype(np.float64)


def _small_cases():
    cases = []
    for seed in range(6):
        n_dst = [1, 7, 33, 64, 64, 50][seed]
        n_src = [1, 9, 33, 64, 40, 64][seed]
        e = [3, 20, 150, 400, 300, 0][seed]
        cases.append(synth.random_graph(n_dst, n_src, e, seed + 10, self_loops=True,
                                        multi=True, isolated_tail=seed % 3) + (n_src,))
    return cases


@pytest.mark.parametrize("case", range(6))
@pytest.mark.parametrize("norm", ["none", "right", "both"])
@pytest.mark.parametrize("weighted", [False, True])
def test_p2_brute_gcn(case, norm, weighted):
    rp, ci, n_src = _small_cases()[case]
    X = synth.features(n_src, 5, 5, seed=case)
    ew = synth.edge_weights(len(ci), case + 3) if weighted else None
    Y, _ = oracle.gcn(rp, ci, X, norm, ew=ew, n_src=n_src)
    np.testing.assert_allclose(Y, _brute_gcn(rp, ci, X, norm, n_src, ew), rtol=1e-12, atol=1e-13)


@pytest.mark.parametrize("case", range(6))
@pytest.mark.parametrize("weighted", [False, True])
def test_p2_brute_gin(case, weighted):
    rp, ci, n_src = _small_cases()[case]
    n_dst = len(rp) - 1
    if n_dst > n_src:
        pytest.skip("GIN needs n_dst <= n_src")
    X = synth.features(n_src, 4, 6, seed=case)
    ew = synth.edge_weights(len(ci), case + 3) if weighted else None
    eps = 0.37
    Y, _ = oracle.gin(rp, ci, X, eps, ew=ew, F=4)
    A, _ = _dense_adj(rp, ci, n_dst, n_src, ew)
    ref = (1 + eps) * X[:n_dst, :4].astype(np.float64) + A @ X[:, :4].astype(np.float64)
    np.testing.assert_allclose(Y, ref, rtol=1e-12, atol=1e-13)


@pytest.mark.parametrize("case", range(6))
@pytest.mark.parametrize("slope", [0.2, 1.0, 0.0])
def test_p2_brute_gat(case, slope):
    rp, ci, n_src = _small_cases()[case]
    n_dst = len(rp) - 1
    X = synth.features(n_src, 3, 3, seed=case)
    el = synth.normal(n_src, case + 50) * 2
    er = synth.normal(max(n_dst, n_src), case + 60) * 2
    Y, _ = oracle.gat(rp, ci, X, el, er, slope)
    np.testing.assert_allclose(Y, _brute_gat(rp, ci, X, el, er, slope, n_src), rtol=1e-11, atol=1e-13)


def test_p2_rectangular_ld_and_rows_subset():
    rp, ci = synth.random_graph(20, 31, 90, 5)
    Xfull = synth.features(31, 7, 9, seed=1)
    Y, A = oracle.gcn(rp, ci, Xfull, "both", n_src=31, F=7)
    ref = _brute_gcn(rp, ci, Xfull[:, :7], "both", 31)
    np.testing.assert_allclose(Y, ref, rtol=1e-12, atol=1e-13)
    rows = np.array([19, 0, 7, 7], np.int64)
    Ys, As = oracle.gcn(rp, ci, Xfull, "both", rows=rows, n_src=31, F=7)
    np.testing.assert_array_equal(Ys, Y[rows])
    np.testing.assert_array_equal(As, A[rows])


# ---------------------------------------------------------------- P3 --------

@pytest.mark.parametrize("name", ["cora", "pubmed"])
def test_p3_scipy(name):
    sp = pytest.importorskip("scipy.sparse")
    cfg = synth.CONFIGS[name]
    rp, ci = synth.dataset_graph(name, device="cpu")
    n = cfg["n"]
    F = 16
    X = synth.features(n, F, F, seed=7)
    ew = synth.edge_weights(len(ci), 8)
    M = sp.csr_matrix((ew.astype(np.float64), ci, rp), shape=(n, n))
    Y, _ = oracle.gcn(rp, ci, X, "none", ew=ew)
    np.testing.assert_allclose(Y, M @ X.astype(np.float64), rtol=1e-12, atol=1e-12)
    deg = np.diff(rp).astype(np.float64)
    dout = np.bincount(ci, minlength=n).astype(np.float64)
    Mb = sp.diags(1 / np.sqrt(np.maximum(deg, 1))) @ sp.csr_matrix(
        (np.ones(len(ci)), ci, rp), shape=(n, n)) @ sp.diags(1 / np.sqrt(np.maximum(dout, 1)))
    Yb, _ = oracle.gcn(rp, ci, X, "both")
    np.testing.assert_allclose(Yb, Mb @ X.astype(np.float64), rtol=1e-12, atol=1e-12)
    Yg, _ = oracle.gin(rp, ci, X, 0.1)
    Mg = sp.csr_matrix((np.ones(len(ci)), ci, rp), shape=(n, n))
    np.testing.assert_allclose(Yg, 1.1 * X.astype(np.float64) + Mg @ X.astype(np.float64),
                               rtol=1e-12, atol=1e-12)


# ---------------------------------------------------------------- P4/P5 -----

@pytest.fixture(scope="module")
def pub():
    rp, ci = synth.dataset_graph("pubmed", device="cpu")
    return rp, ci, synth.CONFIGS["pubmed"]["n"]


def test_p4_right_of_constant(pub):
    rp, ci, n = pub
    X = np.full((n, 3), 0.7, np.float32)
    Y, _ = oracle.gcn(rp, ci, X, "right")
    deg = np.diff(rp)
    np.testing.assert_allclose(Y[deg > 0], np.float64(np.float32(0.7)), rtol=1e-14)
    assert np.all(Y[deg == 0] == 0)


def test_p4_none_of_ones_is_indegree_exactly(pub):
    rp, ci, n = pub
    Y, _ = oracle.gcn(rp, ci, np.ones((n, 2), np.float32), "none")
    assert np.array_equal(Y[:, 0], np.diff(rp).astype(np.float64))


def test_p4_gat_of_ones_and_p5_alpha_sum(pub):
    rp, ci, n = pub
    el = synth.normal(n, 1) * 3
    er = synth.normal(n, 2) * 3
    Y, _, S = oracle.gat(rp, ci, np.ones((n, 2), np.float32), el, er, 0.2,
                         return_alpha_sum=True)
    deg = np.diff(rp)
    assert np.all(np.abs(S[deg > 0] - 1) <= 1e-12)
    assert np.all(np.abs(Y[deg > 0] - 1) <= 1e-12)


def test_p4_gat_constant_el_is_mean(pub):
    rp, ci, n = pub
    X = synth.features(n, 4, seed=3)
    er = synth.normal(n, 2)
    Ya, _ = oracle.gat(rp, ci, X, np.full(n, 0.3, np.float32), er, 0.2)
    Yr, _ = oracle.gcn(rp, ci, X, "right")
    np.testing.assert_allclose(Ya, Yr, rtol=1e-12, atol=1e-14)


def test_p4_gat_slope1_shift_invariant(pub):
    rp, ci, n = pub
    X = synth.features(n, 4, seed=3)
    el = synth.normal(n, 1)
    Y1, _ = oracle.gat(rp, ci, X, el, synth.normal(n, 2), 1.0)
    Y2, _ = oracle.gat(rp, ci, X, el, synth.normal(n, 9) * 5, 1.0)
    np.testing.assert_allclose(Y1, Y2, rtol=1e-11, atol=1e-14)
    # and with slope != 1 er does matter (guards a dropped LeakyReLU branch)
    Y3, _ = oracle.gat(rp, ci, X, el, synth.normal(n, 2), 0.2)
    Y4, _ = oracle.gat(rp, ci, X, el, synth.normal(n, 9) * 5, 0.2)
    assert np.abs(Y3 - Y4).max() > 1e-3


def test_p4_gin_eps_minus1_is_gcn_none(pub):
    rp, ci, n = pub
    X = synth.features(n, 4, seed=3)
    Yg, _ = oracle.gin(rp, ci, X, -1.0)
    Yn, _ = oracle.gcn(rp, ci, X, "none")
    np.testing.assert_allclose(Yg, Yn, rtol=0, atol=0)


def test_p4_linearity_and_column_independence(pub):
    rp, ci, n = pub
    X1 = synth.features(n, 3, seed=1)
    X2 = synth.features(n, 3, seed=2)
    Y1, _ = oracle.gcn(rp, ci, X1, "both")
    Y2, _ = oracle.gcn(rp, ci, X2, "both")
    Y12, _ = oracle.gcn(rp, ci, (X1 + X2).astype(np.float32), "both")
    # X1 + X2 is rounded to fp32 once: compare with a rounding-level tolerance
    np.testing.assert_allclose(Y12, Y1 + Y2, rtol=1e-6, atol=1e-6)
    for f in range(3):
        Yc, _ = oracle.gcn(rp, ci, np.ascontiguousarray(X1[:, f:f + 1]), "both")
        np.testing.assert_array_equal(Yc[:, 0], Y1[:, f])


def test_p4_permutation_equivariance():
    rp, ci = synth.random_graph(40, 40, 300, 3)
    n = 40
    X = synth.features(n, 3, seed=4)
    el = synth.normal(n, 5); er = synth.normal(n, 6)
    perm = np.random.default_rng(0).permutation(n)  # new id of old vertex i is perm[i]
    inv = np.argsort(perm)
    src = ci.astype(np.int64)
    dst = np.repeat(np.arange(n), np.diff(rp))
    rp2, ci2 = synth.csr_from_edges(n, perm[src], perm[dst])
    X2 = X[inv]
    for fn in ("gcn", "gin", "gat"):
        if fn == "gcn":
            Y, _ = oracle.gcn(rp, ci, X, "both"); Y2, _ = oracle.gcn(rp2, ci2, X2, "both")
        elif fn == "gin":
            Y, _ = oracle.gin(rp, ci, X, 0.1); Y2, _ = oracle.gin(rp2, ci2, X2, 0.1)
        else:
            Y, _ = oracle.gat(rp, ci, X, el, er, 0.2)
            Y2, _ = oracle.gat(rp2, ci2, X2, el[inv], er[inv], 0.2)
        np.testing.assert_allclose(Y2[perm], Y, rtol=1e-12, atol=1e-14)


def test_p4_bound_term_dominates_and_is_tight_for_nonneg(pub):
    rp, ci, n = pub
    X = synth.features(n, 4, seed=3)
    Y, A = oracle.gcn(rp, ci, X, "both")
    assert np.all(A >= np.abs(Y) - 1e-15)
    Xp = synth.features(n, 4, seed=3, low=0.0, high=1.0)
    Yp, Ap = oracle.gcn(rp, ci, Xp, "both")
    np.testing.assert_allclose(Ap, Yp, rtol=1e-15)


def test_tolerance_helper_flags_errors():
    ref = np.array([1.0, 2.0]); A = np.array([1.0, 2.0])
    ok, w = oracle.within_tolerance(ref + 1e-7, ref, A)
    assert ok and w < 1
    ok, w = oracle.within_tolerance(ref + 1e-4, ref, A)
    assert not ok and w > 1
    ok, _ = oracle.within_tolerance(np.array([np.nan, 2.0]), ref, A)
    assert not ok


# ---------------------------------------------------------------- P6 --------

def test_p6_degrees_and_validity(pub):
    rp, ci, n = pub
    din = oracle.in_degree(rp)
    dout = oracle.out_degree(ci, n)
    assert din.sum() == len(ci) == dout.sum()
    assert np.array_equal(dout, np.bincount(ci, minlength=n))
    assert np.array_equal(din, np.diff(rp))
    assert oracle.csr_valid(rp, ci, n)


@pytest.mark.parametrize("bad", ["rowptr0", "nonmono", "last", "colneg", "colbig"])
def test_p6_invalid_csr_detected(bad):
    rp, ci = synth.random_graph(10, 10, 30, 1)
    rp = rp.copy(); ci = ci.copy()
    if bad == "rowptr0":
        rp[0] = 1
    elif bad == "nonmono":
        rp[5] = rp[6] + 1
    elif bad == "last":
        rp[-1] -= 1
    elif bad == "colneg":
        ci[3] = -1
    else:
        ci[3] = 10
    assert not oracle.csr_valid(rp, ci, 10)


@pytest.mark.parametrize("parts", [1, 2, 3, 4, 8])
def test_p6_partition(pub, parts):
    rp, ci, n = pub
    b = oracle.partition(rp, parts)
    E = len(ci)
    ref = np.searchsorted(rp, [(k * E) // parts for k in range(parts + 1)], side="left")
    ref[0] = 0
    ref[-1] = n
    assert b.tolist() == ref.tolist()
    assert b[0] == 0 and b[-1] == n and np.all(np.diff(b) >= 0)
    maxdeg = np.diff(rp).max()
    edges = rp[b[1:]] - rp[b[:-1]]
    assert np.all(edges <= -(-E // parts) + maxdeg)
    # concatenated slices reproduce the CSR
    cat_ci = np.concatenate([ci[rp[b[k]]:rp[b[k + 1]]] for k in range(parts)])
    assert np.array_equal(cat_ci, ci)
    cat_rp = [0]
    for k in range(parts):
        sl = rp[b[k]:b[k + 1] + 1] - rp[b[k]]
        cat_rp += (sl[1:] + cat_rp[-1]).tolist()
    assert cat_rp == rp.tolist()


def test_p6_partition_edge_cases():
    # hub holding more than E/P edges -> empty partitions allowed; b_P = N forced
    rp = np.array([0, 100, 101, 102, 102, 102], np.int64)
    b = oracle.partition(rp, 4)
    assert b.tolist() == [0, 1, 1, 1, 5]
    rp0 = np.zeros(4, np.int64)  # E = 0
    assert oracle.partition(rp0, 3).tolist() == [0, 0, 0, 3]
    assert oracle.partition(np.zeros(1, np.int64), 2).tolist() == [0, 0, 0]


# ---------------------------------------------------- NEXT-1: Sage, multi-head GAT --

def test_p1_star_sage():
    g = _star()
    s = g["without_self_loops"]
    rp, ci = synth.figure1_star(self_loops=False)
    X = np.array(g["x"], np.float32).reshape(-1, 1)
    np.testing.assert_allclose(oracle.sage(rp, ci, X)[0].ravel(), s["sage_mean"], rtol=1e-15)
    np.testing.assert_allclose(oracle.sage(rp, ci, X, include_self=True)[0].ravel(),
                               s["sage_mean_with_self"], rtol=1e-15)


@pytest.mark.parametrize("case", range(6))
@pytest.mark.parametrize("include_self", [False, True])
def test_p2_brute_sage(case, include_self):
    rp, ci, n_src = _small_cases()[case]
    n_dst = len(rp) - 1
    if include_self and n_dst > n_src:
        pytest.skip("self row needs n_dst <= n_src")
    X = synth.features(n_src, 5, 6, seed=case)
    Y, _ = oracle.sage(rp, ci, X, include_self=include_self, F=5)
    _, C = _dense_adj(rp, ci, n_dst, n_src)
    if include_self:
        C[np.arange(n_dst), np.arange(n_dst)] += 1
    cnt = np.maximum(C.sum(1, keepdims=True), 1)
    np.testing.assert_allclose(Y, (C / cnt) @ X[:, :5].astype(np.float64), rtol=1e-12, atol=1e-13)


def test_p4_sage_without_self_is_gcn_right(pub):
    rp, ci, n = pub
    X = synth.features(n, 6, seed=8)
    np.testing.assert_allclose(oracle.sage(rp, ci, X)[0], oracle.gcn(rp, ci, X, "right")[0],
                               rtol=1e-14, atol=1e-15)


@pytest.mark.parametrize("case", range(6))
@pytest.mark.parametrize("H,Fh", [(1, 3), (2, 2), (4, 1), (3, 5)])
def test_p2_brute_gat_mh(case, H, Fh):
    rp, ci, n_src = _small_cases()[case]
    n_dst = len(rp) - 1
    X = synth.features(n_src, H * Fh, H * Fh + 1, seed=case)
    el = (synth.normal(n_src * H, case + 70) * 2).reshape(n_src, H)
    er = (synth.normal(max(n_dst, n_src) * H, case + 80) * 2).reshape(-1, H)
    Y, _ = oracle.gat_mh(rp, ci, X, el, er, H, 0.2, Fh=Fh)
    for h in range(H):
        ref = _brute_gat(rp, ci, X[:, h * Fh:(h + 1) * Fh], el[:, h].copy(), er[:, h].copy(), 0.2, n_src)
        np.testing.assert_allclose(Y[:, h * Fh:(h + 1) * Fh], ref, rtol=1e-11, atol=1e-13)


def test_p4_gat_mh_one_head_and_head_permutation(pub):
    rp, ci, n = pub
    X = synth.features(n, 12, seed=4)
    el1, er1 = synth.normal(n, 1), synth.normal(n, 2)
    np.testing.assert_array_equal(oracle.gat_mh(rp, ci, X, el1, er1, 1, 0.2)[0],
                                  oracle.gat(rp, ci, X, el1, er1, 0.2)[0])
    H, Fh = 3, 4
    el = synth.normal(n * H, 5).reshape(n, H)
    er = synth.normal(n * H, 6).reshape(n, H)
    Y = oracle.gat_mh(rp, ci, X, el, er, H, 0.2)[0]
    perm = [2, 0, 1]
    Xp = np.concatenate([X[:, p * Fh:(p + 1) * Fh] for p in perm], axis=1)
    Yp = oracle.gat_mh(rp, ci, Xp, el[:, perm], er[:, perm], H, 0.2)[0]
    np.testing.assert_array_equal(Yp, np.concatenate([Y[:, p * Fh:(p + 1) * Fh] for p in perm], axis=1))


# ---------------------------------------------------- NEXT-3: layer epilogue ---

def test_epilogue_closed_forms():
    Y = np.array([[-2.0, -0.5, 0.0, 0.5, 3.0]])
    A = np.abs(Y)
    b = np.array([0.5, 0.5, 0.0, -1.0, 0.0], np.float32)
    # identity without bias is a no-op
    Yi, Ai = oracle.epilogue(Y, A)
    assert np.array_equal(Yi, Y) and np.array_equal(Ai, A)
    # bias only: y + b, bound gains |b|
    Yb, Ab = oracle.epilogue(Y, A, bias=b)
    assert Yb.tolist() == [[-1.5, 0.0, 0.0, -0.5, 3.0]]
    assert Ab.tolist() == [[2.5, 1.0, 0.0, 1.5, 3.0]]
    # ReLU, LeakyReLU(0.1), ELU(1.0) worked by hand on y + b
    assert oracle.epilogue(Y, A, b, "relu")[0].tolist() == [[0.0, 0.0, 0.0, 0.0, 3.0]]
    np.testing.assert_allclose(oracle.epilogue(Y, A, b, "leaky_relu", 0.1)[0],
                               [[-0.15, 0.0, 0.0, -0.05, 3.0]], rtol=1e-15)
    np.testing.assert_allclose(oracle.epilogue(Y, A, b, "elu", 1.0)[0],
                               [[math.exp(-1.5) - 1, 0.0, 0.0, math.exp(-0.5) - 1, 3.0]], rtol=1e-15)


def test_epilogue_matches_numpy_definitions():
    rng = np.random.default_rng(3)
    Y = rng.standard_normal((50, 7))
    A = np.abs(Y) + 1
    b = rng.standard_normal(7).astype(np.float32)
    x = Y + b.astype(np.float64)
    np.testing.assert_array_equal(oracle.epilogue(Y, A, b, "relu")[0], np.maximum(x, 0))
    np.testing.assert_array_equal(oracle.epilogue(Y, A, b, "leaky_relu", 0.2)[0], np.where(x >= 0, x, 0.2 * x))
    np.testing.assert_allclose(oracle.epilogue(Y, A, b, "elu", 0.7)[0], np.where(x > 0, x, 0.7 * np.expm1(x)),
                               rtol=1e-14, atol=1e-16)


# ---------------------------------------------------- NEXT-4: backward ---------

@pytest.mark.parametrize("case", range(6))
@pytest.mark.parametrize("norm", ["none", "right", "both"])
@pytest.mark.parametrize("weighted", [False, True])
def test_p2_brute_gcn_backward(case, norm, weighted):
    rp, ci, n_src = _small_cases()[case]
    n_dst = len(rp) - 1
    dY = synth.features(n_dst, 4, 5, seed=case + 40)
    ew = synth.edge_weights(len(ci), case + 3) if weighted else None
    dX, _ = oracle.gcn_backward(rp, ci, dY, norm, ew=ew, n_src=n_src, F=4)
    # dense operator M from the forward brute force, applied transposed
    M = _brute_gcn(rp, ci, np.eye(n_src, dtype=np.float32), norm, n_src, ew)
    np.testing.assert_allclose(dX, M.T @ dY[:, :4].astype(np.float64), rtol=1e-12, atol=1e-13)


@pytest.mark.parametrize("norm", ["none", "right", "both"])
def test_p4_gcn_adjoint_identity(pub, norm):
    """<M X, G> = <X, M^T G> (exact up to fp64 rounding)."""
    rp, ci, n = pub
    X = synth.features(n, 3, seed=1)
    G = synth.features(n, 3, seed=2)
    Y, _ = oracle.gcn(rp, ci, X, norm)
    dX, _ = oracle.gcn_backward(rp, ci, G, norm)
    lhs = float((Y * G.astype(np.float64)).sum())
    rhs = float((X.astype(np.float64) * dX).sum())
    assert abs(lhs - rhs) <= 1e-9 * (abs(lhs) + 1)


@pytest.mark.parametrize("case", [1, 2, 3, 5])
def test_p2_brute_gin_backward(case):
    rp, ci, n_src = _small_cases()[case]
    n = len(rp) - 1
    if n != n_src:
        pytest.skip("square graphs only")
    dY = synth.features(n, 4, 4, seed=case)
    ew = synth.edge_weights(len(ci), 2)
    dX, _ = oracle.gin_backward(rp, ci, dY, 0.3, ew=ew)
    A, _ = _dense_adj(rp, ci, n, n, ew)
    np.testing.assert_allclose(dX, 1.3 * dY.astype(np.float64) + A.T @ dY.astype(np.float64),
                               rtol=1e-12, atol=1e-13)


# ---------------------------------------------------- NEXT-4: GAT backward -----

def test_gat_backward_hand_worked():
    """One destination with two sources, el = er = 0 (alpha = 1/2 each), F = 1,
    X = [1, 3], dY = 1:  g = [1, 3], S = 2, ds = [-1/2, 1/2]; t = 0 >= 0 so
    dt = ds;  del = [-1/2, 1/2], der = 0, dX = [1/2, 1/2]."""
    rp = np.array([0, 2, 2, 2], dtype=np.int64)
    ci = np.array([1, 2], dtype=np.int32)
    X = np.array([[0.0], [1.0], [3.0]], dtype=np.float32)
    z = np.zeros(3, dtype=np.float32)
    dY = np.array([[1.0], [0.0], [0.0]], dtype=np.float32)
    (dX, _), (dl, _), (dr, _) = oracle.gat_backward(rp, ci, X, z, z, 0.2, dY)
    np.testing.assert_allclose(dX[:, 0], [0.0, 0.5, 0.5], atol=1e-15)
    np.testing.assert_allclose(dl, [0.0, -0.5, 0.5], atol=1e-15)
    np.testing.assert_allclose(dr, [0.0, 0.0, 0.0], atol=1e-15)


def _torch_dense_gat_grads(rp, ci, X, el, er, slope, dY, n_src):
    """Autograd (torch, fp64, CPU) of L = <Y, dY> for the dense masked-softmax
    GAT (multi-edges weighted by their count): a library routine independent of
    the oracle's hand-written chain rule."""
    import torch
    n_dst = len(rp) - 1
    _, C = _dense_adj(rp, ci, n_dst, n_src)
    Ct = torch.tensor(C, dtype=torch.float64)
    Xt = torch.tensor(X.astype(np.float64), requires_grad=True)
    elt = torch.tensor(el.astype(np.float64), requires_grad=True)
    ert = torch.tensor(er.astype(np.float64)[:n_dst], requires_grad=True)
    T = ert[:, None] + elt[None, :]
    S = torch.where(T >= 0, T, slope * T)
    mask = Ct > 0
    Sm = torch.where(mask, S, torch.full_like(S, -1e300))
    m = Sm.max(1, keepdim=True).values.detach()
    P = torch.where(mask, Ct * torch.exp(torch.where(mask, S - m, torch.zeros_like(S))),
                    torch.zeros_like(S))
    Z = P.sum(1, keepdim=True)
    P = P / torch.where(Z > 0, Z, torch.ones_like(Z))
    Y = P @ Xt
    (Y * torch.tensor(dY.astype(np.float64))).sum().backward()
    return Xt.grad.numpy(), elt.grad.numpy(), ert.grad.numpy()


@pytest.mark.parametrize("case", range(6))
@pytest.mark.parametrize("slope", [0.2, 1.0, 0.0])
def test_p2_autograd_gat_backward(case, slope):
    rp, ci, n_src = _small_cases()[case]
    n_dst = len(rp) - 1
    F = 5
    X = synth.features(n_src, F, seed=case + 60)
    el = synth.normal(n_src, case + 61)
    er = synth.normal(n_dst, case + 62)
    dY = synth.features(n_dst, F, seed=case + 63)
    (dX, AdX), (dl, Adl), (dr, Adr) = oracle.gat_backward(rp, ci, X, el, er, slope, dY)
    tX, tl, tr = _torch_dense_gat_grads(rp, ci, X, el, er, slope, dY, n_src)
    np.testing.assert_allclose(dX, tX, rtol=1e-11, atol=1e-13)
    np.testing.assert_allclose(dl, tl, rtol=1e-10, atol=1e-12)
    np.testing.assert_allclose(dr, tr, rtol=1e-10, atol=1e-12)
    # bound terms dominate the values
    assert np.all(np.abs(dX) <= AdX + 1e-15) and np.all(np.abs(dl) <= Adl + 1e-15)
    assert np.all(np.abs(dr) <= Adr + 1e-15)


def test_p4_gat_backward_invariants(pub):
    """sum_v der = sum_u del (both are sum_e dt_e); slope = 1 gives der = 0
    (softmax gradients sum to zero over a row, shift invariance); dX of
    constant-score rows is the GCN-RIGHT transpose; <Y, G> = <X, dX> (Y is
    linear in X for fixed scores)."""
    rp, ci, n = pub
    F = 3
    X = synth.features(n, F, seed=5)
    el = synth.normal(n, 6)
    er = synth.normal(n, 7)
    G = synth.features(n, F, seed=8)
    (dX, _), (dl, Adl), (dr, Adr) = oracle.gat_backward(rp, ci, X, el, er, 0.2, G)
    assert abs(dl.sum() - dr.sum()) <= 1e-9 * (Adl.sum() + 1)
    Y, _ = oracle.gat(rp, ci, X, el, er, 0.2)
    assert abs(float((Y * G.astype(np.float64)).sum()) -
               float((X.astype(np.float64) * dX).sum())) <= 1e-9 * (np.abs(Y).sum() + 1)
    (_, _), (_, _), (dr1, Adr1) = oracle.gat_backward(rp, ci, X, el, er, 1.0, G)
    assert np.all(np.abs(dr1) <= 1e-12 * (Adr1 + 1))
    z = np.zeros(n, dtype=np.float32)
    (dXc, _), _, _ = oracle.gat_backward(rp, ci, X, z, z, 0.2, G)
    dXr, _ = oracle.gcn_backward(rp, ci, G, "right")
    np.testing.assert_allclose(dXc, dXr, rtol=1e-12, atol=1e-14)


def test_gat_backward_finite_differences():
    """Central differences of L = <GAT(X, el, er), dY> in fp64 (the dense
    forward, h = 1e-6) against the oracle's del / der."""
    rp, ci, n_src = _small_cases()[2]
    n_dst = len(rp) - 1
    X = synth.features(n_src, 4, seed=70)
    el = synth.normal(n_src, 71).astype(np.float64)
    er = synth.normal(n_dst, 72).astype(np.float64)
    dY = synth.features(n_dst, 4, seed=73).astype(np.float64)
    (_, _), (dl, _), (dr, _) = oracle.gat_backward(rp, ci, X, el.astype(np.float32),
                                                   er.astype(np.float32), 0.2, dY.astype(np.float32))

    def loss(el_, er_):
        return float((_brute_gat(rp, ci, X, el_, er_, 0.2, n_src) * dY).sum())

    h = 1e-6
    for u in range(0, n_src, 5):
        ep, em = el.copy(), el.copy()
        ep[u] += h
        em[u] -= h
        assert abs((loss(ep, er) - loss(em, er)) / (2 * h) - dl[u]) <= 1e-6 * (abs(dl[u]) + 1)
    for v in range(0, n_dst, 5):
        ep, em = er.copy(), er.copy()
        ep[v] += h
        em[v] -= h
        assert abs((loss(el, ep) - loss(el, em)) / (2 * h) - dr[v]) <= 1e-6 * (abs(dr[v]) + 1)


# ------------------------------------------------- NEXT-3: epilogue projections --

def test_project_closed_forms():
    """Unit vector e_k picks column k exactly; ones give the row sum; the star's
    GCN-NONE output [10, 3, 4, 5] (F = 1) times a = 0.5 is [5, 1.5, 2, 2.5]."""
    Y = synth.features(50, 7, 9, seed=3)
    for k in range(7):
        e = np.zeros(7, np.float32)
        e[k] = 1.0
        out, A = oracle.project(Y, e, F=7)
        np.testing.assert_array_equal(out, Y[:, k].astype(np.float64))
        np.testing.assert_array_equal(A, np.abs(Y[:, k].astype(np.float64)))
    out, _ = oracle.project(Y, np.ones(7, np.float32), F=7)
    np.testing.assert_allclose(out, Y[:, :7].astype(np.float64).sum(1), rtol=1e-13)
    rp, ci = synth.figure1_star(self_loops=True)
    Ys, _ = oracle.gcn(rp, ci, np.array([[1.0], [2.0], [3.0], [4.0]], np.float32), "none")
    out, _ = oracle.project(Ys.astype(np.float32), np.array([0.5], np.float32))
    np.testing.assert_allclose(out, [5.0, 1.5, 2.0, 2.5], rtol=0, atol=0)

"""Pins of the oracle's bound outputs A = sum|terms| (column
"A64"; the north-star criterion |err| <= 1e-5*A + 1e-6 hangs on them).

Every parity tolerance is derived from A, so each A is fixed here by something
other than the oracle's own loops:

* the Figure-1 star with MIXED-SIGN x = [1, -2, 3, -4] worked by hand
  (tests/golden/figure1_star.json "mixed_sign"):
  with x of both signs A differs from |Y| and from sum|X|, so a bound that drops
  alpha (GAT), c_out / c_in (GCN), the (1+eps) factor (GIN) or the 1/count
  (SAGE) fails;
* dense brute force on <= 64-vertex graphs with multi-edges, self-loops and
  isolated rows: A = |M| |X| with M the dense operator of each op
  (GCN diag(c_in) Adj diag(c_out); GIN |1+eps| I + |Adj|; GAT / GAT-mh the
  dense softmax matrix P per head; SAGE C / count) and, for the backward ops,
  |M|^T |dY| and the dense form of the dt-bound.
"""
import json
import os

import numpy as np
import pytest

import oracle
import synth

GOLD = os.path.join(os.path.dirname(__file__), "golden", "figure1_star.json")


def _mixed():
    with open(GOLD) as f:
        return json.load(f)["mixed_sign"]


def _x(g):
    return np.array(g["x"], np.float32).reshape(-1, 1)


# ---------------------------------------------------------------- hand-worked --

@pytest.mark.parametrize("norm", ["none", "right", "both"])
def test_star_mixed_gcn_value_and_bound(norm):
    g = _mixed()
    rp, ci = synth.figure1_star(self_loops=True)
    Y, A = oracle.gcn(rp, ci, _x(g), norm)
    np.testing.assert_allclose(Y.ravel(), g["gcn_" + norm], rtol=1e-14, atol=1e-15)
    np.testing.assert_allclose(A.ravel(), g["A_gcn_" + norm], rtol=1e-14)


def test_star_mixed_gin_value_and_bound():
    g = _mixed()
    rp, ci = synth.figure1_star(self_loops=False)
    Y, A = oracle.gin(rp, ci, _x(g), 0.5)
    np.testing.assert_allclose(Y.ravel(), g["gin_eps0.5"], rtol=1e-15)
    np.testing.assert_allclose(A.ravel(), g["A_gin_eps0.5"], rtol=1e-15)
    # eps = -3 makes the self coefficient negative: the bound takes |1+eps|
    Y, A = oracle.gin(rp, ci, _x(g), -3.0)
    np.testing.assert_allclose(Y.ravel(), g["gin_eps-3"], rtol=1e-15)
    np.testing.assert_allclose(A.ravel(), g["A_gin_eps-3"], rtol=1e-15)


def test_star_mixed_gat_value_and_bound():
    g = _mixed()
    rp, ci = synth.figure1_star(self_loops=True)
    el = np.log(np.abs(np.array(g["x"], np.float64))).astype(np.float32)
    er = np.zeros(4, np.float32)
    Y, A = oracle.gat(rp, ci, _x(g), el, er, 0.2)
    # el = ln|x| rounded to fp32 perturbs alpha by ~1e-7 (relative)
    np.testing.assert_allclose(Y.ravel(), g["gat_el_ln|x|_er0"], rtol=1e-6)
    np.testing.assert_allclose(A.ravel(), g["A_gat_el_ln|x|_er0"], rtol=1e-6)


def test_star_mixed_sage_value_and_bound():
    g = _mixed()
    rp, ci = synth.figure1_star(self_loops=False)
    Y, A = oracle.sage(rp, ci, _x(g), include_self=True)
    np.testing.assert_allclose(Y.ravel(), g["sage_mean_with_self"], rtol=1e-15)
    np.testing.assert_allclose(A.ravel(), g["A_sage_mean_with_self"], rtol=1e-15)
    Y, A = oracle.sage(rp, ci, _x(g))
    np.testing.assert_allclose(Y.ravel(), g["sage_mean"], rtol=1e-15)
    np.testing.assert_allclose(A.ravel(), g["A_sage_mean"], rtol=1e-15)


def test_star_mixed_gat_mh_bound():
    """Two heads: head 0 is the single-head case above (el = ln|x|), head 1 has
    constant scores (uniform alpha = mean); column 1 holds x as well."""
    g = _mixed()
    rp, ci = synth.figure1_star(self_loops=True)
    x = np.array(g["x"], np.float32)
    X = np.stack([x, x], axis=1)
    el = np.stack([np.log(np.abs(x.astype(np.float64))).astype(np.float32), np.zeros(4, np.float32)], 1)
    er = np.zeros((4, 2), np.float32)
    Y, A = oracle.gat_mh(rp, ci, X, el, er, 2, 0.2)
    np.testing.assert_allclose(Y[:, 0], g["gat_el_ln|x|_er0"], rtol=1e-6)
    np.testing.assert_allclose(A[:, 0], g["A_gat_el_ln|x|_er0"], rtol=1e-6)
    np.testing.assert_allclose(Y[:, 1], g["gcn_right"], rtol=1e-14)
    np.testing.assert_allclose(A[:, 1], g["A_gcn_right"], rtol=1e-14)


def test_star_mixed_gcn_backward_bound():
    """The star with self-loops is symmetric, so with NONE the transpose
    product equals the forward one: dX = Adj dY, A = Adj |dY|."""
    g = _mixed()
    rp, ci = synth.figure1_star(self_loops=True)
    dX, A = oracle.gcn_backward(rp, ci, _x(g), "none")
    np.testing.assert_allclose(dX.ravel(), g["gcn_none"], rtol=1e-15)
    np.testing.assert_allclose(A.ravel(), g["A_gcn_none"], rtol=1e-15)


def test_two_edge_gat_backward_bounds_hand_worked():
    """One destination (row 0) with sources 1, 2; el = er = 0 so alpha = 1/2;
    F = 2, X[1] = [1, -1], X[2] = [3, 2], dY[0] = [1, -2]:
      g = [1*1 + (-2)(-1), 1*3 + (-2)(2)] = [3, -1],  G = [|1|+|2|, |3|+|4|] = [3, 7]
      S = (3 - 1)/2 = 1,  SA = (3 + 7)/2 = 5;  t = 0 >= 0 so lr = 1
      dt = alpha (g - S) = [1, -1];  B = alpha (G + SA) = [4, 6]
      del = [0, 1, -1], Adel = [0, 4, 6];  der[0] = 0, Ader[0] = 10
      dX[1] = dX[2] = dY/2 = [0.5, -1],  AdX = [0.5, 1]."""
    rp = np.array([0, 2, 2, 2], dtype=np.int64)
    ci = np.array([1, 2], dtype=np.int32)
    X = np.array([[0, 0], [1, -1], [3, 2]], dtype=np.float32)
    z = np.zeros(3, dtype=np.float32)
    dY = np.array([[1, -2], [0, 0], [0, 0]], dtype=np.float32)
    (dX, AdX), (dl, Adl), (dr, Adr) = oracle.gat_backward(rp, ci, X, z, z, 0.2, dY)
    np.testing.assert_allclose(dl, [0, 1, -1], atol=1e-15)
    np.testing.assert_allclose(Adl, [0, 4, 6], atol=1e-15)
    np.testing.assert_allclose(dr, [0, 0, 0], atol=1e-15)
    np.testing.assert_allclose(Adr, [10, 0, 0], atol=1e-15)
    np.testing.assert_allclose(dX, [[0, 0], [0.5, -1], [0.5, -1]], atol=1e-15)
    np.testing.assert_allclose(AdX, [[0, 0], [0.5, 1], [0.5, 1]], atol=1e-15)
    # negative scores: slope enters the bound as |slope|
    el = np.array([0, -1, -1], np.float32)
    (_, _), (dl2, Adl2), (_, _) = oracle.gat_backward(rp, ci, X, el, z, 0.2, dY)
    np.testing.assert_allclose(dl2, [0, 0.2, -0.2], atol=1e-15)
    np.testing.assert_allclose(Adl2, [0, 0.8, 1.2], atol=1e-15)


# ---------------------------------------------------------------- dense brute --

def _cases():
    out = []
    for seed in range(6):
        n_dst = [1, 7, 33, 64, 64, 50][seed]
        n_src = [1, 9, 33, 64, 40, 64][seed]
        e = [3, 20, 150, 400, 300, 0][seed]
        out.append(synth.random_graph(n_dst, n_src, e, seed + 10, self_loops=True,
                                      multi=True, isolated_tail=seed % 3) + (n_src,))
    return out


def _counts(rp, ci, n_dst, n_src, ew=None):
    """Adj[v,u] = sum of w_e over u->v, C[v,u] = edge count (multi-edges add)."""
    Adj = np.zeros((n_dst, n_src))
    C = np.zeros((n_dst, n_src))
    for v in range(n_dst):
        for e in range(rp[v], rp[v + 1]):
            Adj[v, ci[e]] += 1.0 if ew is None else float(ew[e])
            C[v, ci[e]] += 1.0
    return Adj, C


def _dense_softmax(C, el, er, slope):
    n_dst = C.shape[0]
    T = er.astype(np.float64)[:n_dst, None] + el.astype(np.float64)[None, :]
    S = np.where(T >= 0, T, slope * T)
    S = np.where(C > 0, S, -np.inf)
    m = S.max(1, keepdims=True)
    m = np.where(np.isfinite(m), m, 0.0)
    P = C * np.exp(S - m)
    Z = P.sum(1, keepdims=True)
    return np.divide(P, Z, out=np.zeros_like(P), where=Z > 0), T


def _mixed_weights(n, seed):
    """Edge weights of both signs (the bound must take |w|)."""
    return (synth.edge_weights(n, seed) * np.where(np.arange(n) % 3 == 1, -1, 1)).astype(np.float32)


@pytest.mark.parametrize("case", range(6))
@pytest.mark.parametrize("norm", ["none", "right", "both"])
@pytest.mark.parametrize("weighted", [False, True])
def test_brute_gcn_bound(case, norm, weighted):
    rp, ci, n_src = _cases()[case]
    n_dst = len(rp) - 1
    X = synth.features(n_src, 5, 5, seed=case)
    ew = _mixed_weights(len(ci), case + 3) if weighted else None
    _, A = oracle.gcn(rp, ci, X, norm, ew=ew, n_src=n_src)
    Adj, C = _counts(rp, ci, n_dst, n_src, None if ew is None else np.abs(ew))
    din, dout = C.sum(1), C.sum(0)
    if norm == "none":
        cin, cout = np.ones(n_dst), np.ones(n_src)
    elif norm == "right":
        cin, cout = 1.0 / np.maximum(din, 1), np.ones(n_src)
    else:
        cin, cout = 1.0 / np.sqrt(np.maximum(din, 1)), 1.0 / np.sqrt(np.maximum(dout, 1))
    ref = (cin[:, None] * Adj * cout[None, :]) @ np.abs(X.astype(np.float64))
    np.testing.assert_allclose(A, ref, rtol=1e-12, atol=1e-14)


@pytest.mark.parametrize("case", range(6))
@pytest.mark.parametrize("eps", [0.37, -2.5])
@pytest.mark.parametrize("weighted", [False, True])
def test_brute_gin_bound(case, eps, weighted):
    rp, ci, n_src = _cases()[case]
    n_dst = len(rp) - 1
    if n_dst > n_src:
        pytest.skip("GIN needs n_dst <= n_src")
    X = synth.features(n_src, 4, 6, seed=case)
    ew = _mixed_weights(len(ci), case + 3) if weighted else None
    _, A = oracle.gin(rp, ci, X, eps, ew=ew, F=4)
    Adj, _ = _counts(rp, ci, n_dst, n_src, None if ew is None else np.abs(ew))
    aX = np.abs(X[:, :4].astype(np.float64))
    np.testing.assert_allclose(A, abs(1 + eps) * aX[:n_dst] + Adj @ aX, rtol=1e-12, atol=1e-14)


@pytest.mark.parametrize("case", range(6))
@pytest.mark.parametrize("slope", [0.2, 1.0])
def test_brute_gat_bound(case, slope):
    rp, ci, n_src = _cases()[case]
    n_dst = len(rp) - 1
    X = synth.features(n_src, 3, 3, seed=case)
    el = synth.normal(n_src, case + 50) * 2
    er = synth.normal(max(n_dst, n_src), case + 60) * 2
    _, A = oracle.gat(rp, ci, X, el, er, slope)
    _, C = _counts(rp, ci, n_dst, n_src)
    P, _ = _dense_softmax(C, el, er, slope)
    np.testing.assert_allclose(A, P @ np.abs(X.astype(np.float64)), rtol=1e-11, atol=1e-14)


@pytest.mark.parametrize("case", range(6))
@pytest.mark.parametrize("include_self", [False, True])
def test_brute_sage_bound(case, include_self):
    rp, ci, n_src = _cases()[case]
    n_dst = len(rp) - 1
    if include_self and n_dst > n_src:
        pytest.skip("self row needs n_dst <= n_src")
    X = synth.features(n_src, 5, 6, seed=case)
    _, A = oracle.sage(rp, ci, X, include_self=include_self, F=5)
    _, C = _counts(rp, ci, n_dst, n_src)
    if include_self:
        C[np.arange(n_dst), np.arange(n_dst)] += 1
    cnt = np.maximum(C.sum(1, keepdims=True), 1)
    np.testing.assert_allclose(A, (C / cnt) @ np.abs(X[:, :5].astype(np.float64)), rtol=1e-12, atol=1e-14)


@pytest.mark.parametrize("case", range(6))
@pytest.mark.parametrize("H,Fh", [(2, 2), (3, 5)])
def test_brute_gat_mh_bound(case, H, Fh):
    rp, ci, n_src = _cases()[case]
    n_dst = len(rp) - 1
    X = synth.features(n_src, H * Fh, H * Fh + 1, seed=case)
    el = (synth.normal(n_src * H, case + 70) * 2).reshape(n_src, H)
    er = (synth.normal(max(n_dst, n_src) * H, case + 80) * 2).reshape(-1, H)
    _, A = oracle.gat_mh(rp, ci, X, el, er, H, 0.2, Fh=Fh)
    _, C = _counts(rp, ci, n_dst, n_src)
    for h in range(H):
        P, _ = _dense_softmax(C, el[:, h], er[:, h], 0.2)
        ref = P @ np.abs(X[:, h * Fh:(h + 1) * Fh].astype(np.float64))
        np.testing.assert_allclose(A[:, h * Fh:(h + 1) * Fh], ref, rtol=1e-11, atol=1e-14)


@pytest.mark.parametrize("case", range(6))
@pytest.mark.parametrize("norm", ["none", "right", "both"])
def test_brute_gcn_backward_bound(case, norm):
    rp, ci, n_src = _cases()[case]
    n_dst = len(rp) - 1
    dY = synth.features(n_dst, 4, 5, seed=case + 40)
    ew = _mixed_weights(len(ci), case + 3)
    _, A = oracle.gcn_backward(rp, ci, dY, norm, ew=ew, n_src=n_src, F=4)
    Adj, C = _counts(rp, ci, n_dst, n_src, np.abs(ew))
    din, dout = C.sum(1), C.sum(0)
    if norm == "none":
        cin, cout = np.ones(n_dst), np.ones(n_src)
    elif norm == "right":
        cin, cout = 1.0 / np.maximum(din, 1), np.ones(n_src)
    else:
        cin, cout = 1.0 / np.sqrt(np.maximum(din, 1)), 1.0 / np.sqrt(np.maximum(dout, 1))
    M = cin[:, None] * Adj * cout[None, :]
    np.testing.assert_allclose(A, M.T @ np.abs(dY[:, :4].astype(np.float64)), rtol=1e-12, atol=1e-14)


@pytest.mark.parametrize("case", [1, 2, 3, 5])
@pytest.mark.parametrize("eps", [0.3, -1.7])
def test_brute_gin_backward_bound(case, eps):
    rp, ci, n_src = _cases()[case]
    n = len(rp) - 1
    if n != n_src:
        pytest.skip("square graphs only")
    dY = synth.features(n, 4, 4, seed=case)
    ew = _mixed_weights(len(ci), 2)
    _, A = oracle.gin_backward(rp, ci, dY, eps, ew=ew)
    Adj, _ = _counts(rp, ci, n, n, np.abs(ew))
    adY = np.abs(dY.astype(np.float64))
    np.testing.assert_allclose(A, abs(1 + eps) * adY + Adj.T @ adY, rtol=1e-12, atol=1e-14)


@pytest.mark.parametrize("case", range(6))
@pytest.mark.parametrize("slope", [0.2, -0.5])
def test_brute_gat_backward_bounds(case, slope):
    """AdX = P^T |dY|; with G[v,u] = sum_f |dY[v,f] X[u,f]| = (|dY| |X|^T)[v,u],
    SA_v = sum_u P[v,u] G[v,u] and the per-(v,u) edge bound
    B[v,u] = |lr(t_vu)| P[v,u] (G[v,u] + SA_v) (P sums the alphas of multi-edges):
    Ader = B.sum(1), Adel = B.sum(0)."""
    rp, ci, n_src = _cases()[case]
    n_dst = len(rp) - 1
    F = 5
    X = synth.features(n_src, F, seed=case + 60)
    el = synth.normal(n_src, case + 61)
    er = synth.normal(n_dst, case + 62)
    dY = synth.features(n_dst, F, seed=case + 63)
    (_, AdX), (_, Adl), (_, Adr) = oracle.gat_backward(rp, ci, X, el, er, slope, dY)
    _, C = _counts(rp, ci, n_dst, n_src)
    P, T = _dense_softmax(C, el, er, slope)
    adY = np.abs(dY.astype(np.float64))
    aX = np.abs(X.astype(np.float64))
    G = adY @ aX.T
    SA = (P * G).sum(1, keepdims=True)
    lr = np.where(T >= 0, 1.0, abs(slope))
    B = lr * P * (G + SA)
    np.testing.assert_allclose(AdX, P.T @ adY, rtol=1e-11, atol=1e-14)
    np.testing.assert_allclose(Adr, B.sum(1), rtol=1e-11, atol=1e-14)
    np.testing.assert_allclose(Adl, B.sum(0), rtol=1e-11, atol=1e-14)


def test_project_bound_mixed_sign():
    """el[v] = Y[v] . a; A = |Y| . |a| (hand-worked: Y = [1, -2], a = [3, 1]:
    value 1, bound 5)."""
    Y = np.array([[1.0, -2.0]], np.float32)
    a = np.array([3.0, 1.0], np.float32)
    out, A = oracle.project(Y, a)
    assert out.tolist() == [1.0] and A.tolist() == [5.0]


# ---------------------------------------------------------------- row slices ---

@pytest.mark.parametrize("case", [2, 3, 4])
def test_brute_row_slice_row_offset(case):
    """A destination-row slice [b, b+m) with its rebased CSR and row_offset = b
    (the dist layout, c1 "Partition") equals rows [b, b+m) of the dense brute
    force of the whole graph, for the ops that read per-row inputs at
    row_offset + v (GAT er, GIN / SAGE self rows)."""
    rp, ci, n_src = _cases()[case]
    n_dst = len(rp) - 1
    if n_dst > n_src:
        pytest.skip("self rows need n_dst <= n_src")
    b, m = n_dst // 3, n_dst // 3
    srp = (rp[b:b + m + 1] - rp[b]).astype(np.int64)
    sci = ci[rp[b]:rp[b + m]]
    X = synth.features(n_src, 3, 3, seed=case)
    el = synth.normal(n_src, case + 50) * 2
    er = synth.normal(n_src, case + 60) * 2
    Adj, C = _counts(rp, ci, n_dst, n_src)
    x64 = X.astype(np.float64)
    P, _ = _dense_softmax(C, el, er, 0.2)
    Y, A = oracle.gat(srp, sci, X, el, er, 0.2, row_offset=b)
    np.testing.assert_allclose(Y, (P @ x64)[b:b + m], rtol=1e-11, atol=1e-14)
    np.testing.assert_allclose(A, (P @ np.abs(x64))[b:b + m], rtol=1e-11, atol=1e-14)
    Y, A = oracle.gin(srp, sci, X, 0.3, row_offset=b)
    np.testing.assert_allclose(Y, (1.3 * x64[:n_dst] + Adj @ x64)[b:b + m], rtol=1e-12, atol=1e-14)
    Cs = C.copy()
    Cs[np.arange(n_dst), np.arange(n_dst)] += 1
    cnt = np.maximum(Cs.sum(1, keepdims=True), 1)
    Y, _ = oracle.sage(srp, sci, X, include_self=True, row_offset=b)
    np.testing.assert_allclose(Y, ((Cs / cnt) @ x64)[b:b + m], rtol=1e-12, atol=1e-14)

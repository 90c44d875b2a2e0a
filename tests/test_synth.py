"""The seeded generators deliver the pre-registered recipe."""
import numpy as np
import pytest

import synth


def _check_symmetric_simple(rp, ci, n):
    assert rp[0] == 0 and np.all(np.diff(rp) >= 0) and rp[-1] == len(ci)
    dst = np.repeat(np.arange(n, dtype=np.int64), np.diff(rp))
    src = ci.astype(np.int64)
    assert np.all(src != dst), "self-loop"
    key = dst * n + src
    assert np.all(np.diff(key) > 0), "CSR not sorted by (dst, src) or multi-edge"
    rkey = np.sort(src * n + dst)
    assert np.array_equal(rkey, key), "not symmetric"


@pytest.mark.parametrize("name", ["cora", "pubmed"])
def test_chung_lu_exact_counts(name):
    cfg = synth.CONFIGS[name]
    rp, ci = synth.chung_lu(cfg["n"], cfg["e"], cfg["alpha"], cfg["seed"], device="cpu")
    assert len(rp) == cfg["n"] + 1 and len(ci) == cfg["e"]
    _check_symmetric_simple(rp, ci, cfg["n"])
    st = synth.degree_stats(rp)
    # power-law: the max degree is far above the mean (logged in DESIGN.md)
    assert st["max"] > 10 * st["mean"]


def test_chung_lu_deterministic():
    a = synth.chung_lu(500, 4000, 0.5, 11, device="cpu")
    b = synth.chung_lu(500, 4000, 0.5, 11, device="cpu")
    c = synth.chung_lu(500, 4000, 0.5, 12, device="cpu")
    assert np.array_equal(a[0], b[0]) and np.array_equal(a[1], b[1])
    assert not np.array_equal(a[1], c[1])


def test_rmat_small():
    rp, ci = synth.rmat(10, 8, 5, device="cpu")
    n = 1 << 10
    assert len(ci) == 2 * 8 * n
    _check_symmetric_simple(rp, ci, n)
    rp2, ci2 = synth.rmat(10, 8, 5, device="cpu")
    assert np.array_equal(ci, ci2)


def test_features_recipe():
    X = synth.features(100, 7, 9, seed=3)
    assert X.dtype == np.float32 and X.shape == (100, 9)
    assert np.all(X[:, 7:] == 0)
    assert X[:, :7].min() >= -1 and X[:, :7].max() < 1
    Xp = synth.features(100, 7, 7, seed=3, low=0.0, high=1.0)
    assert Xp.min() >= 0
    assert np.array_equal(synth.features(10, 3, seed=1), synth.features(10, 3, seed=1))
    w = synth.edge_weights(1000, 1)
    assert w.min() > 0 and w.max() <= 1


def test_small_graph_helpers():
    rp, ci = synth.random_graph(10, 12, 50, 1, isolated_tail=3)
    assert np.all(np.diff(rp)[-3:] == 0) and len(ci) == 50
    assert ci.max() < 12
    rp, ci = synth.power_law_rows(4, [0, 5, 1, 0], 7, 2)
    assert rp.tolist() == [0, 0, 5, 6, 6]

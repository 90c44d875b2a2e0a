"""fp64 CPU oracle for the TLPGNN aggregation hot path -- TEST INFRASTRUCTURE ONLY.

Only ``tests/``, ``__graft_entry__.smoke()`` and ``bench.py``'s ``cpu_baseline`` /
``--impl reference`` legs may import this package.  The product package
(``paper_conf_hpdc_fujh22_b200``) never imports it, and it never imports the
product package: the two share no code.

The arithmetic lives in ``tlp_oracle.c`` (plain single-threaded fp64 CSR
loops, one function per operation, each citing PAPER.md).  This module only
compiles it with gcc and marshals numpy arrays through ctypes.

Parity pins (tests/test_oracle_pins.py) tie every function here to something
other than itself: the Figure-1 star worked by hand (tests/golden), dense
brute force, scipy.sparse, closed-form invariants.  Nothing is "parity
unpinned" except the absolute values of the paper, which prints none
(SURVEY 8(c) c3).
"""
from __future__ import annotations

import ctypes
import os
import subprocess

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "tlp_oracle.c")
_LIB_PATH = os.path.join(_HERE, "liboracle.so")
_lib = None

NORM_NONE, NORM_RIGHT, NORM_BOTH = 0, 1, 2
_NORMS = {"none": NORM_NONE, "right": NORM_RIGHT, "both": NORM_BOTH}


def build(force: bool = False) -> str:
    """Compile tlp_oracle.c into liboracle.so (gcc, -O2, no fast-math, no FMA
    contraction: plain IEEE double)."""
    if force or not os.path.exists(_LIB_PATH) or (
            os.path.getmtime(_LIB_PATH) < os.path.getmtime(_SRC)):
        tmp = _LIB_PATH + ".tmp%d" % os.getpid()
        subprocess.check_call([
            "gcc", "-O2", "-std=c99", "-fPIC", "-shared", "-ffp-contract=off",
            "-fno-fast-math", "-o", tmp, _SRC, "-lm"])
        os.replace(tmp, _LIB_PATH)
    return _LIB_PATH


def _load():
    global _lib
    if _lib is None:
        build()
        lib = ctypes.CDLL(_LIB_PATH)
        P = ctypes.c_void_p
        I64 = ctypes.c_int64
        lib.oracle_in_degree.argtypes = [I64, P, P]
        lib.oracle_out_degree.argtypes = [I64, I64, P, P]
        lib.oracle_csr_invalid.argtypes = [I64, I64, I64, P, P]
        lib.oracle_csr_invalid.restype = ctypes.c_int
        lib.oracle_partition.argtypes = [I64, P, ctypes.c_int, P]
        lib.oracle_gcn.argtypes = [I64, I64, P, P, P, P, I64, I64, ctypes.c_int,
                                   I64, P, P, P]
        lib.oracle_gcn.restype = ctypes.c_int
        lib.oracle_gin.argtypes = [I64, I64, P, P, P, P, I64, I64, ctypes.c_double,
                                   I64, I64, P, P, P]
        lib.oracle_gin.restype = ctypes.c_int
        lib.oracle_gat.argtypes = [I64, I64, P, P, P, I64, I64, P, P,
                                   ctypes.c_double, I64, I64, P, P, P, P]
        lib.oracle_gat.restype = ctypes.c_int
        lib.oracle_sage.argtypes = [I64, I64, P, P, P, I64, I64, ctypes.c_int, I64, I64, P, P, P]
        lib.oracle_sage.restype = ctypes.c_int
        lib.oracle_gat_mh.argtypes = [I64, I64, P, P, P, I64, I64, I64, P, P, ctypes.c_double,
                                      I64, I64, P, P, P]
        lib.oracle_gat_mh.restype = ctypes.c_int
        lib.oracle_epilogue.argtypes = [I64, I64, P, P, P, ctypes.c_int, ctypes.c_double]
        lib.oracle_epilogue.restype = ctypes.c_int
        lib.oracle_gcn_backward.argtypes = [I64, I64, P, P, P, P, I64, I64, ctypes.c_int, P, P]
        lib.oracle_gcn_backward.restype = ctypes.c_int
        lib.oracle_gin_backward.argtypes = [I64, P, P, P, P, I64, I64, ctypes.c_double, P, P]
        lib.oracle_gin_backward.restype = ctypes.c_int
        lib.oracle_gat_backward.argtypes = [I64, I64, P, P, P, I64, P, P, ctypes.c_double, P,
                                            I64, I64, P, P, P, P, P, P]
        lib.oracle_gat_backward.restype = ctypes.c_int
        lib.oracle_project.argtypes = [I64, I64, P, I64, P, P, P]
        lib.oracle_project.restype = ctypes.c_int
        _lib = lib
    return _lib


def _ptr(a):
    return None if a is None else a.ctypes.data_as(ctypes.c_void_p)


def _csr(rowptr, colidx):
    rowptr = np.ascontiguousarray(rowptr, dtype=np.int64)
    colidx = np.ascontiguousarray(colidx, dtype=np.int32)
    return rowptr, colidx


def _feat(X):
    X = np.asarray(X, dtype=np.float32)
    if X.ndim == 1:
        X = X.reshape(-1, 1)
    if X.strides[1] != 4 or X.strides[0] % 4:
        X = np.ascontiguousarray(X)
    return X


def _rows(rows, n_dst):
    if rows is None:
        return None, n_dst
    rows = np.ascontiguousarray(rows, dtype=np.int64)
    return rows, rows.shape[0]


def in_degree(rowptr):
    rowptr = np.ascontiguousarray(rowptr, dtype=np.int64)
    n = rowptr.shape[0] - 1
    out = np.empty(n, np.int32)
    _load().oracle_in_degree(n, _ptr(rowptr), _ptr(out))
    return out


def out_degree(colidx, n_src):
    colidx = np.ascontiguousarray(colidx, dtype=np.int32)
    out = np.empty(n_src, np.int32)
    _load().oracle_out_degree(n_src, colidx.shape[0], _ptr(colidx), _ptr(out))
    return out


def csr_valid(rowptr, colidx, n_src):
    rowptr, colidx = _csr(rowptr, colidx)
    n = rowptr.shape[0] - 1
    return _load().oracle_csr_invalid(n, n_src, colidx.shape[0], _ptr(rowptr),
                                      _ptr(colidx)) == 0


def partition(rowptr, parts):
    rowptr = np.ascontiguousarray(rowptr, dtype=np.int64)
    n = rowptr.shape[0] - 1
    b = np.empty(parts + 1, np.int64)
    _load().oracle_partition(n, _ptr(rowptr), int(parts), _ptr(b))
    return b


def gcn(rowptr, colidx, X, norm="both", ew=None, rows=None, n_src=None, F=None):
    """Returns (Y, A) as float64 [n_rows, F]; X is fp32 [n_src, ld >= F]."""
    rowptr, colidx = _csr(rowptr, colidx)
    X = _feat(X)
    n_dst = rowptr.shape[0] - 1
    n_src = X.shape[0] if n_src is None else n_src
    F = X.shape[1] if F is None else F
    ldx = X.strides[0] // 4
    ew = None if ew is None else np.ascontiguousarray(ew, dtype=np.float32)
    rows, nr = _rows(rows, n_dst)
    Y = np.empty((nr, F)); A = np.empty((nr, F))
    rc = _load().oracle_gcn(n_dst, n_src, _ptr(rowptr), _ptr(colidx), _ptr(ew),
                            _ptr(X), F, ldx, _NORMS.get(norm, norm), nr, _ptr(rows),
                            _ptr(Y), _ptr(A))
    if rc:
        raise ValueError("oracle_gcn: bad arguments")
    return Y, A


def gin(rowptr, colidx, X, eps, ew=None, rows=None, row_offset=0, F=None):
    rowptr, colidx = _csr(rowptr, colidx)
    X = _feat(X)
    n_dst = rowptr.shape[0] - 1
    n_src = X.shape[0]
    F = X.shape[1] if F is None else F
    ldx = X.strides[0] // 4
    ew = None if ew is None else np.ascontiguousarray(ew, dtype=np.float32)
    rows, nr = _rows(rows, n_dst)
    Y = np.empty((nr, F)); A = np.empty((nr, F))
    rc = _load().oracle_gin(n_dst, n_src, _ptr(rowptr), _ptr(colidx), _ptr(ew),
                            _ptr(X), F, ldx, float(eps), int(row_offset), nr,
                            _ptr(rows), _ptr(Y), _ptr(A))
    if rc:
        raise ValueError("oracle_gin: bad arguments")
    return Y, A


def gat(rowptr, colidx, X, el, er, slope, rows=None, row_offset=0, F=None,
        return_alpha_sum=False):
    rowptr, colidx = _csr(rowptr, colidx)
    X = _feat(X)
    n_dst = rowptr.shape[0] - 1
    n_src = X.shape[0]
    F = X.shape[1] if F is None else F
    ldx = X.strides[0] // 4
    el = np.ascontiguousarray(el, dtype=np.float32)
    er = np.ascontiguousarray(er, dtype=np.float32)
    rows, nr = _rows(rows, n_dst)
    Y = np.empty((nr, F)); A = np.empty((nr, F)); S = np.empty(nr)
    rc = _load().oracle_gat(n_dst, n_src, _ptr(rowptr), _ptr(colidx), _ptr(X), F,
                            ldx, _ptr(el), _ptr(er), float(slope), int(row_offset),
                            nr, _ptr(rows), _ptr(Y), _ptr(A), _ptr(S))
    if rc:
        raise ValueError("oracle_gat: bad arguments")
    return (Y, A, S) if return_alpha_sum else (Y, A)


def sage(rowptr, colidx, X, include_self=False, rows=None, row_offset=0, F=None):
    """GraphSage mean (optionally including the self row).  Returns (Y, A)."""
    rowptr, colidx = _csr(rowptr, colidx)
    X = _feat(X)
    n_dst = rowptr.shape[0] - 1
    F = X.shape[1] if F is None else F
    ldx = X.strides[0] // 4
    rows, nr = _rows(rows, n_dst)
    Y = np.empty((nr, F)); A = np.empty((nr, F))
    rc = _load().oracle_sage(n_dst, X.shape[0], _ptr(rowptr), _ptr(colidx), _ptr(X), F, ldx,
                             int(bool(include_self)), int(row_offset), nr, _ptr(rows), _ptr(Y),
                             _ptr(A))
    if rc:
        raise ValueError("oracle_sage: bad arguments")
    return Y, A


def gat_mh(rowptr, colidx, X, el, er, heads, slope, rows=None, row_offset=0, Fh=None):
    """Multi-head GAT: el, er are [n, heads] (row-major); head h owns columns
    [h*Fh, (h+1)*Fh).  Returns (Y, A) of width heads*Fh."""
    rowptr, colidx = _csr(rowptr, colidx)
    X = _feat(X)
    n_dst = rowptr.shape[0] - 1
    H = int(heads)
    Fh = X.shape[1] // H if Fh is None else int(Fh)
    ldx = X.strides[0] // 4
    el = np.ascontiguousarray(el, dtype=np.float32).reshape(-1)
    er = np.ascontiguousarray(er, dtype=np.float32).reshape(-1)
    rows, nr = _rows(rows, n_dst)
    Y = np.empty((nr, H * Fh)); A = np.empty((nr, H * Fh))
    rc = _load().oracle_gat_mh(n_dst, X.shape[0], _ptr(rowptr), _ptr(colidx), _ptr(X), H, Fh, ldx,
                               _ptr(el), _ptr(er), float(slope), int(row_offset), nr, _ptr(rows),
                               _ptr(Y), _ptr(A))
    if rc:
        raise ValueError("oracle_gat_mh: bad arguments")
    return Y, A


def gcn_backward(rowptr, colidx, dY, norm="both", ew=None, n_src=None, F=None):
    """dX = M^T dY for the GCN operator M (returns (dX, A) [n_src, F])."""
    rowptr, colidx = _csr(rowptr, colidx)
    dY = _feat(dY)
    n_dst = rowptr.shape[0] - 1
    n_src = n_dst if n_src is None else n_src
    F = dY.shape[1] if F is None else F
    ew = None if ew is None else np.ascontiguousarray(ew, dtype=np.float32)
    dX = np.empty((n_src, F)); A = np.empty((n_src, F))
    rc = _load().oracle_gcn_backward(n_dst, n_src, _ptr(rowptr), _ptr(colidx), _ptr(ew), _ptr(dY), F,
                                     dY.strides[0] // 4, _NORMS.get(norm, norm), _ptr(dX), _ptr(A))
    if rc:
        raise ValueError("oracle_gcn_backward: bad arguments")
    return dX, A


def gin_backward(rowptr, colidx, dY, eps, ew=None, F=None):
    rowptr, colidx = _csr(rowptr, colidx)
    dY = _feat(dY)
    n = rowptr.shape[0] - 1
    F = dY.shape[1] if F is None else F
    ew = None if ew is None else np.ascontiguousarray(ew, dtype=np.float32)
    dX = np.empty((n, F)); A = np.empty((n, F))
    rc = _load().oracle_gin_backward(n, _ptr(rowptr), _ptr(colidx), _ptr(ew), _ptr(dY), F,
                                     dY.strides[0] // 4, float(eps), _ptr(dX), _ptr(A))
    if rc:
        raise ValueError("oracle_gin_backward: bad arguments")
    return dX, A


def gat_backward(rowptr, colidx, X, el, er, slope, dY, F=None):
    """Single-head GAT backward.  Returns ((dX, AdX), (del, Adel), (der, Ader)):
    dX [n_src, F], del [n_src], der [n_dst] with their sum|terms| bounds."""
    rowptr, colidx = _csr(rowptr, colidx)
    X = _feat(X)
    dY = _feat(dY)
    n_dst = rowptr.shape[0] - 1
    n_src = X.shape[0]
    F = X.shape[1] if F is None else F
    el = np.ascontiguousarray(el, dtype=np.float32)
    er = np.ascontiguousarray(er, dtype=np.float32)
    dX = np.empty((n_src, F)); AdX = np.empty((n_src, F))
    dl = np.empty(n_src); Adl = np.empty(n_src)
    dr = np.empty(n_dst); Adr = np.empty(n_dst)
    rc = _load().oracle_gat_backward(n_dst, n_src, _ptr(rowptr), _ptr(colidx), _ptr(X),
                                     X.strides[0] // 4, _ptr(el), _ptr(er), float(slope), _ptr(dY),
                                     F, dY.strides[0] // 4, _ptr(dX), _ptr(AdX), _ptr(dl),
                                     _ptr(Adl), _ptr(dr), _ptr(Adr))
    if rc:
        raise ValueError("oracle_gat_backward: bad arguments")
    return (dX, AdX), (dl, Adl), (dr, Adr)


def project(Y, a, F=None):
    """el[v] = sum_f Y[v,f] a[f] for an fp32 layer output Y.  Returns (el, A)."""
    Y = _feat(Y)
    F = Y.shape[1] if F is None else F
    a = np.ascontiguousarray(a, dtype=np.float32)
    out = np.empty(Y.shape[0]); A = np.empty(Y.shape[0])
    rc = _load().oracle_project(Y.shape[0], F, _ptr(Y), Y.strides[0] // 4, _ptr(a), _ptr(out), _ptr(A))
    if rc:
        raise ValueError("oracle_project: bad arguments")
    return out, A


ACTS = {"none": 0, "relu": 1, "leaky_relu": 2, "elu": 3}


def epilogue(Y, A, bias=None, act="none", param=0.0):
    """Layer epilogue h' = act(Y + bias) applied to oracle outputs (returns copies)."""
    Y = np.ascontiguousarray(Y, dtype=np.float64).copy()
    A = np.ascontiguousarray(A, dtype=np.float64).copy()
    n, F = Y.shape
    b = None if bias is None else np.ascontiguousarray(bias, dtype=np.float32)
    rc = _load().oracle_epilogue(n, F, _ptr(Y), _ptr(A), _ptr(b), ACTS.get(act, act), float(param))
    if rc:
        raise ValueError("oracle_epilogue: bad arguments")
    return Y, A


def within_tolerance(Y_test, Y_ref, A_ref, rel=1e-5, abs_=1e-6):
    """The north-star parity criterion |err| <= 1e-5*sum|terms| + 1e-6, per element.
    Returns (ok, worst ratio err/tol)."""
    Y_test = np.asarray(Y_test, dtype=np.float64)
    err = np.abs(Y_test - Y_ref)
    tol = rel * A_ref + abs_
    ratio = err / tol
    worst = float(np.nanmax(ratio)) if ratio.size else 0.0
    ok = bool(np.all(err <= tol)) and not np.isnan(Y_test).any()
    return ok, worst

"""Thin Python binding of libtlp (the C ABI in include/tlp.h).

Argument marshalling only: every step of the aggregation path runs in the
CUDA kernels of libtlp.so (paper_conf_hpdc_fujh22_b200/csrc).  There is no CPU
fallback -- importing this package fails loudly when the library is missing,
and the aggregation calls reject non-CUDA feature tensors.

The function names are the C ABI's (``tlp_graph_create``, ``tlp_gcn_aggregate``
...).  ``Graph`` is a small convenience wrapper around a handle.

PyTorch supplies device memory, the current CUDA stream and (for the dist
layer) the process group that broadcasts the NCCL unique id; it never computes
any part of the path.
"""
from __future__ import annotations

import ctypes
import os

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
# TLP_LIB_PATH selects an in-tree tuning variant of the library (bench/profiling)
LIB_PATH = os.environ.get("TLP_LIB_PATH") or os.path.join(_HERE, "libtlp.so")

if not os.path.exists(LIB_PATH):
    raise ImportError(
        f"{LIB_PATH} is missing: build it with `python -c 'import __graft_entry__ as g; g.build()'` "
        "(there is no CPU fallback)")

_lib = ctypes.CDLL(LIB_PATH)

# ------------------------------------------------------------------ C types --
TLP_OK = 0
STATUS = {0: "TLP_OK", 1: "TLP_ERR_INVALID_ARGUMENT", 2: "TLP_ERR_INVALID_GRAPH",
          3: "TLP_ERR_OUT_OF_MEMORY", 4: "TLP_ERR_CUDA", 5: "TLP_ERR_NCCL",
          6: "TLP_ERR_UNSUPPORTED"}
NORMS = {"none": 0, "right": 1, "both": 2}
SCHEDS = {"dynamic": 0, "static": 1, "hardware": 2, "paper": 3, "clc": 4}


class tlp_create_opts(ctypes.Structure):
    _fields_ = [("hub_threshold", ctypes.c_int64), ("hub_chunk", ctypes.c_int64),
                ("unit_edges", ctypes.c_int64)]


class tlp_graph_info(ctypes.Structure):
    _fields_ = [(n, ctypes.c_int64) for n in (
        "n_dst", "n_src", "nnz", "row_offset", "max_in_degree", "n_hubs", "n_hub_chunks",
        "n_units", "n_tasks", "hub_threshold", "hub_chunk", "unit_edges", "has_edge_weight",
        "device_bytes", "scratch_bytes")] + [("create_ms", ctypes.c_double),
                                             ("launches", ctypes.c_int64)]


class tlp_agg_desc(ctypes.Structure):
    _fields_ = [("op", ctypes.c_int), ("X", ctypes.c_void_p), ("F", ctypes.c_int64),
                ("ldx", ctypes.c_int64), ("Y", ctypes.c_void_p), ("ldy", ctypes.c_int64),
                ("norm", ctypes.c_int), ("eps", ctypes.c_float), ("el", ctypes.c_void_p),
                ("er", ctypes.c_void_p), ("slope", ctypes.c_float), ("heads", ctypes.c_int64),
                ("include_self", ctypes.c_int), ("bias", ctypes.c_void_p), ("act", ctypes.c_int),
                ("act_param", ctypes.c_float), ("att_l", ctypes.c_void_p), ("att_r", ctypes.c_void_p),
                ("el_out", ctypes.c_void_p), ("er_out", ctypes.c_void_p)]


OPS = {"gcn": 0, "gin": 1, "gat": 2, "sage": 3, "gat_mh": 4}
ACTS = {"none": 0, "relu": 1, "leaky_relu": 2, "elu": 3}

_P = ctypes.c_void_p
_I64 = ctypes.c_int64
_I = ctypes.c_int
_F = ctypes.c_float
_sig = {
    "tlp_status_string": ([_I], ctypes.c_char_p),
    "tlp_last_error": ([], ctypes.c_char_p),
    "tlp_version": ([], _I),
    "tlp_graph_create": ([_I64, _I64, _I64, _P, _P, _P, _P, ctypes.POINTER(_P)], _I),
    "tlp_graph_create_ex": ([_I64, _I64, _I64, _P, _P, _P, ctypes.POINTER(tlp_create_opts), _P,
                             ctypes.POINTER(_P)], _I),
    "tlp_graph_destroy": ([_P], _I),
    "tlp_graph_info_get": ([_P, ctypes.POINTER(tlp_graph_info)], _I),
    "tlp_graph_degrees": ([_P, _P, _P, _P], _I),
    "tlp_graph_plan": ([_P, _P, _P, _P, _P], _I),
    "tlp_graph_set_schedule": ([_P, _I, _I, _I], _I),
    "tlp_graph_set_visit_counter": ([_P, _P], _I),
    "tlp_graph_build_transpose": ([_P, _P], _I),
    "tlp_gcn_backward": ([_P, _P, _I64, _I64, _I, _P, _I64, _P], _I),
    "tlp_gin_backward": ([_P, _P, _I64, _I64, _F, _P, _I64, _P], _I),
    "tlp_gat_backward": ([_P, _P, _I64, _I64, _P, _P, _F, _P, _I64, _P, _I64, _P, _I64, _P, _P, _P],
                         _I),
    "tlp_gcn_aggregate": ([_P, _P, _I64, _I64, _I, _P, _I64, _P], _I),
    "tlp_gin_aggregate": ([_P, _P, _I64, _I64, _F, _P, _I64, _P], _I),
    "tlp_gat_aggregate": ([_P, _P, _I64, _I64, _P, _P, _F, _P, _I64, _P], _I),
    "tlp_sage_aggregate": ([_P, _P, _I64, _I64, _I, _P, _I64, _P], _I),
    "tlp_aggregate": ([_P, ctypes.POINTER(tlp_agg_desc), _P], _I),
    "tlp_dist_aggregate": ([_P, _P, ctypes.POINTER(tlp_agg_desc), _P], _I),
    "tlp_gat_mh_aggregate": ([_P, _P, _I64, _I64, _I64, _P, _P, _F, _P, _I64, _P], _I),
    "tlp_graph_create_rows": ([_I64, _I64, _P, _P, _P, _I64, _I64, ctypes.POINTER(tlp_create_opts),
                               _P, ctypes.POINTER(_P)], _I),
    "tlp_partition_rows": ([_P, _I64, _I, _P], _I),
    "tlp_comm_get_unique_id": ([_P], _I),
    "tlp_comm_create": ([_P, _I, _I, ctypes.POINTER(_P)], _I),
    "tlp_comm_destroy": ([_P], _I),
    "tlp_comm_async_error": ([_P, ctypes.POINTER(_I)], _I),
    "tlp_comm_abort": ([_P], _I),
    "tlp_comm_wait": ([_P, _P, ctypes.c_double], _I),
    "tlp_dist_graph_create": ([_P, _I64, _I64, _P, _P, _P, ctypes.POINTER(tlp_create_opts), _P,
                               ctypes.POINTER(_P)], _I),
    "tlp_dist_bounds": ([_P, _P], _I),
    "tlp_comm_alloc_symmetric": ([_P, ctypes.c_size_t, ctypes.POINTER(_P)], _I),
    "tlp_comm_free_symmetric": ([_P, _P], _I),
    "tlp_comm_symmetric_kind": ([_P, _P, ctypes.POINTER(_I)], _I),
    "tlp_dist_aggregate_fused": ([_P, _P, ctypes.POINTER(tlp_agg_desc), _P], _I),
    "tlp_debug_multi_store": ([_P, ctypes.POINTER(tlp_agg_desc), _P, _I, _P], _I),
    "tlp_dist_allgather_rows": ([_P, _P, _P, _I64, _P], _I),
    "tlp_dist_gcn_aggregate": ([_P, _P, _P, _I64, _I64, _I, _P, _I64, _P], _I),
    "tlp_dist_gin_aggregate": ([_P, _P, _P, _I64, _I64, _F, _P, _I64, _P], _I),
    "tlp_dist_gat_aggregate": ([_P, _P, _P, _I64, _I64, _P, _P, _F, _P, _I64, _P], _I),
    "tlp_dist_sage_aggregate": ([_P, _P, _P, _I64, _I64, _I, _P, _I64, _P], _I),
    "tlp_dist_gat_mh_aggregate": ([_P, _P, _P, _I64, _I64, _I64, _P, _P, _F, _P, _I64, _P], _I),
}
for _name, (_args, _res) in _sig.items():
    _fn = getattr(_lib, _name)
    _fn.argtypes = _args
    _fn.restype = _res

C_SYMBOLS = tuple(_sig)


class TlpError(RuntimeError):
    def __init__(self, status, where):
        self.status = status
        detail = _lib.tlp_last_error().decode(errors="replace")
        super().__init__(f"{where}: {STATUS.get(status, status)}: {detail}")


def _check(st, where):
    if st != TLP_OK:
        raise TlpError(st, where)


def tlp_version():
    return _lib.tlp_version()


def tlp_status_string(s):
    return _lib.tlp_status_string(s).decode()


# --------------------------------------------------------------- marshalling --

def _torch():
    import torch
    return torch


def _ptr(a):
    """Raw pointer of a torch tensor / numpy array (host or device) or None."""
    if a is None:
        return None
    if isinstance(a, np.ndarray):
        return a.ctypes.data
    return a.data_ptr()


def _as_index(a, dtype):
    """Keep torch tensors (any device) as they are if contiguous and of the right
    dtype; numpy goes through as host memory (the library copies it)."""
    torch = _torch()
    if isinstance(a, torch.Tensor):
        a = a.contiguous()
        want = torch.int64 if dtype == np.int64 else (torch.int32 if dtype == np.int32 else torch.float32)
        return a if a.dtype == want else a.to(want)
    return np.ascontiguousarray(a, dtype=dtype)


def _stream(stream, device=None):
    """cudaStream_t of `stream`, or torch's current stream on `device` (the raw
    handle straight from torch's C layer: this runs once per call, so it
    avoids building a Stream object)."""
    if stream is not None:
        return getattr(stream, "cuda_stream", stream)
    torch = _torch()
    if torch.cuda.is_available():
        idx = device.index if device is not None and device.index is not None else torch.cuda.current_device()
        raw = getattr(torch._C, "_cuda_getCurrentRawStream", None)
        return raw(idx) if raw is not None else torch.cuda.current_stream(idx).cuda_stream
    return None


def _feat(X, F):
    torch = _torch()
    if not isinstance(X, torch.Tensor) or not X.is_cuda:
        raise TypeError("features must be a CUDA torch tensor (no CPU fallback)")
    if X.dtype != torch.float32:
        raise TypeError("features must be float32")
    if X.dim() == 1:
        X = X.view(-1, 1)
    if X.dim() != 2 or (X.shape[1] > 1 and X.stride(1) != 1) or X.stride(0) < 1:
        raise ValueError("features must be a row-major 2-D tensor with unit column stride")
    F = X.shape[1] if F is None else int(F)
    ld = X.stride(0) if X.shape[0] > 1 else max(X.stride(0), X.shape[1])
    if F > ld:
        raise ValueError("F exceeds the leading dimension")
    return X, F, ld


def _out(Y, n, F, like):
    torch = _torch()
    if Y is None:
        ld = (F + 3) // 4 * 4 if F > 0 else 1
        buf = torch.empty((n, ld), dtype=torch.float32, device=like.device)
        return buf[:, :F], F, ld
    Y, F2, ldy = _feat(Y, F)
    return Y, F, ldy


def _vec_cuda(v, name, n=None):
    """A float32 CUDA vector of at least n elements.  A non-contiguous input is
    copied; the copy is registered with the launch stream by _keep_alive so the
    caching allocator cannot recycle it while the kernel is queued."""
    torch = _torch()
    if not isinstance(v, torch.Tensor) or not v.is_cuda or v.dtype != torch.float32:
        raise TypeError(f"{name} must be a float32 CUDA tensor")
    if n is not None and v.numel() < n:
        raise ValueError(f"{name} has {v.numel()} elements, the call reads {n}")
    return v.contiguous()


def _keep_alive(stream_handle, *tensors):
    """Tie temporaries passed to a kernel to the stream the kernel was enqueued
    on (no-op when that is torch's current stream: the allocator already
    orders reuse on it)."""
    torch = _torch()
    for t in tensors:
        if t is None or not isinstance(t, torch.Tensor) or not t.is_cuda:
            continue
        if stream_handle is None or stream_handle == torch.cuda.current_stream(t.device).cuda_stream:
            continue
        t.record_stream(torch.cuda.ExternalStream(stream_handle, device=t.device))


def _need_rows(T, n, name):
    if T.shape[0] < n:
        raise ValueError(f"{name} has {T.shape[0]} rows, the graph needs {n}")


# ------------------------------------------------------------------ graph ----

def tlp_graph_create(rowptr, colidx, n_src=None, edge_weight=None, opts=None, stream=None):
    """Returns an opaque handle (int).  rowptr/colidx/edge_weight: torch tensors
    (CUDA or CPU) or numpy arrays."""
    rowptr = _as_index(rowptr, np.int64)
    colidx = _as_index(colidx, np.int32)
    ew = None if edge_weight is None else _as_index(edge_weight, np.float32)
    n_dst = int(rowptr.shape[0]) - 1
    nnz = int(colidx.shape[0])
    if ew is not None and int(ew.shape[0]) != nnz:
        raise ValueError(f"edge_weight has {int(ew.shape[0])} entries, colidx has {nnz}")
    if n_src is None:
        n_src = n_dst
    out = _P()
    if opts:
        o = tlp_create_opts(int(opts.get("hub_threshold", 0)), int(opts.get("hub_chunk", 0)),
                            int(opts.get("unit_edges", 0)))
        st = _lib.tlp_graph_create_ex(n_dst, int(n_src), nnz, _ptr(rowptr), _ptr(colidx), _ptr(ew),
                                      ctypes.byref(o), _stream(stream), ctypes.byref(out))
    else:
        st = _lib.tlp_graph_create(n_dst, int(n_src), nnz, _ptr(rowptr), _ptr(colidx), _ptr(ew),
                                   _stream(stream), ctypes.byref(out))
    _check(st, "tlp_graph_create")
    return out.value


def _opts(opts):
    if not opts:
        return None
    return tlp_create_opts(int(opts.get("hub_threshold", 0)), int(opts.get("hub_chunk", 0)),
                           int(opts.get("unit_edges", 0)))


def tlp_graph_create_rows(rowptr, colidx, row_begin, row_end, edge_weight=None, opts=None,
                          stream=None):
    """Handle for rows [row_begin, row_end) of the full square CSR (global
    sources and out-degrees, row_offset = row_begin)."""
    rowptr = _as_index(rowptr, np.int64)
    colidx = _as_index(colidx, np.int32)
    ew = None if edge_weight is None else _as_index(edge_weight, np.float32)
    n = int(rowptr.shape[0]) - 1
    out = _P()
    o = _opts(opts)
    st = _lib.tlp_graph_create_rows(n, int(colidx.shape[0]), _ptr(rowptr), _ptr(colidx), _ptr(ew),
                                    int(row_begin), int(row_end), ctypes.byref(o) if o else None,
                                    _stream(stream), ctypes.byref(out))
    _check(st, "tlp_graph_create_rows")
    return out.value


def tlp_graph_destroy(g):
    _check(_lib.tlp_graph_destroy(g), "tlp_graph_destroy")


def tlp_graph_info_get(g):
    info = tlp_graph_info()
    _check(_lib.tlp_graph_info_get(g, ctypes.byref(info)), "tlp_graph_info_get")
    return {n: getattr(info, n) for n, _ in info._fields_}


def tlp_graph_degrees(g, stream=None):
    info = tlp_graph_info_get(g)
    din = np.empty(info["n_dst"], np.int32)
    dout = np.empty(info["n_src"], np.int32)
    _check(_lib.tlp_graph_degrees(g, _ptr(din), _ptr(dout), _stream(stream)), "tlp_graph_degrees")
    return din, dout


def tlp_graph_plan(g, stream=None):
    info = tlp_graph_info_get(g)
    tasks = np.empty((info["n_tasks"], 2), np.int32)
    hubs = np.empty(info["n_hubs"], np.int32)
    off = np.empty(info["n_hubs"] + 1, np.int32)
    _check(_lib.tlp_graph_plan(g, _ptr(tasks), _ptr(hubs), _ptr(off), _stream(stream)),
           "tlp_graph_plan")
    return tasks, hubs, off


def tlp_graph_set_schedule(g, sched="dynamic", warps_per_cta=0, step=0):
    s = SCHEDS[sched] if isinstance(sched, str) else int(sched)
    _check(_lib.tlp_graph_set_schedule(g, s, int(warps_per_cta), int(step)),
           "tlp_graph_set_schedule")


def tlp_graph_set_visit_counter(g, counter=None):
    """Debug: count finished (row, strip) stores into `counter` (int32 CUDA
    tensor [n_dst], zeroed by the caller); None switches it off."""
    torch = _torch()
    if counter is not None and (not isinstance(counter, torch.Tensor) or not counter.is_cuda
                                or counter.dtype != torch.int32 or not counter.is_contiguous()):
        raise TypeError("counter must be a contiguous int32 CUDA tensor")
    _check(_lib.tlp_graph_set_visit_counter(g, _ptr(counter)), "tlp_graph_set_visit_counter")


def tlp_graph_build_transpose(g, stream=None):
    _check(_lib.tlp_graph_build_transpose(g, _stream(stream)), "tlp_graph_build_transpose")


# ------------------------------------------------------------ aggregations ---

def _info(g, info=None):
    return tlp_graph_info_get(g) if info is None else info


def _n_dst(g):
    return tlp_graph_info_get(g)["n_dst"]


def _fwd_args(g, X, Y, F, info):
    """Shape checks of a forward aggregation (the C ABI gets raw pointers and
    cannot check them): X has the graph's n_src rows, Y (if given) n_dst."""
    info = _info(g, info)
    X, F, ldx = _feat(X, F)
    _need_rows(X, info["n_src"], "X")
    Y, F, ldy = _out(Y, info["n_dst"], F, X)
    _need_rows(Y, info["n_dst"], "Y")
    return info, X, F, ldx, Y, ldy


def _gat_vecs(info, el, er, heads=1):
    el = _vec_cuda(el, "el", info["n_src"] * heads)
    er = _vec_cuda(er, "er", (info["row_offset"] + info["n_dst"]) * heads)
    return el, er


def tlp_gcn_aggregate(g, X, norm="both", Y=None, F=None, stream=None, n_dst=None, info=None):
    info, X, F, ldx, Y, ldy = _fwd_args(g, X, Y, F, info)
    nm = NORMS[norm] if isinstance(norm, str) else int(norm)
    _check(_lib.tlp_gcn_aggregate(g, _ptr(X), F, ldx, nm, _ptr(Y), ldy, _stream(stream, X.device)),
           "tlp_gcn_aggregate")
    return Y


def tlp_gin_aggregate(g, X, eps=0.0, Y=None, F=None, stream=None, n_dst=None, info=None):
    info, X, F, ldx, Y, ldy = _fwd_args(g, X, Y, F, info)
    _check(_lib.tlp_gin_aggregate(g, _ptr(X), F, ldx, float(eps), _ptr(Y), ldy,
                                  _stream(stream, X.device)), "tlp_gin_aggregate")
    return Y


def tlp_gat_aggregate(g, X, el, er, slope=0.2, Y=None, F=None, stream=None, n_dst=None, info=None):
    info, X, F, ldx, Y, ldy = _fwd_args(g, X, Y, F, info)
    el, er = _gat_vecs(info, el, er)
    sh = _stream(stream, X.device)
    _check(_lib.tlp_gat_aggregate(g, _ptr(X), F, ldx, _ptr(el), _ptr(er), float(slope), _ptr(Y),
                                  ldy, sh), "tlp_gat_aggregate")
    _keep_alive(sh, el, er)
    return Y


def _desc(op, X, Y, F, ldx, ldy, norm="both", eps=0.0, el=None, er=None, slope=0.2, heads=1,
          include_self=False, bias=None, act="none", act_param=0.0, att_l=None, att_r=None,
          el_out=None, er_out=None):
    d = tlp_agg_desc()
    d.op = OPS[op] if isinstance(op, str) else int(op)
    d.X, d.F, d.ldx, d.Y, d.ldy = _ptr(X), int(F), int(ldx), _ptr(Y), int(ldy)
    d.norm = NORMS[norm] if isinstance(norm, str) else int(norm)
    d.eps, d.slope, d.heads = float(eps), float(slope), int(heads)
    d.el = _ptr(el)
    d.er = _ptr(er)
    d.include_self = int(bool(include_self))
    d.bias = _ptr(bias)
    d.act = ACTS[act] if isinstance(act, str) else int(act)
    d.act_param = float(act_param)
    d.att_l = _ptr(att_l)
    d.att_r = _ptr(att_r)
    d.el_out = _ptr(el_out)
    d.er_out = _ptr(er_out)
    return d


def _desc_vectors(info, op, F, kw, n_rows_global=None):
    """Check and make contiguous the vector arguments of a descriptor call;
    returns the (possibly copied) tensors to keep alive."""
    heads = int(kw.get("heads", 1) or 1)
    n_src = info["n_src"]
    n_er = n_rows_global if n_rows_global is not None else info["row_offset"] + info["n_dst"]
    sizes = {"el": n_src * heads, "er": n_er * heads, "bias": F, "att_l": F, "att_r": F}
    keep = []
    for k, n in sizes.items():
        if kw.get(k) is not None:
            kw[k] = _vec_cuda(kw[k], k, n)
            keep.append(kw[k])
    return keep


def tlp_aggregate(g, op, X, Y=None, F=None, stream=None, n_dst=None, info=None, **kw):
    """Descriptor API: op in {gcn, gin, gat, sage, gat_mh}; keyword arguments of
    tlp_agg_desc (norm, eps, el, er, slope, heads, include_self) plus the fused
    layer epilogue bias=[F] tensor, act in {none, relu, leaky_relu, elu}, act_param,
    and the next layer's attention projections att_l / att_r ([F]) written to
    el_out / er_out ([n_dst] float32 CUDA tensors, contiguous)."""
    info, X, F, ldx, Y, ldy = _fwd_args(g, X, Y, F, info)
    n = info["n_dst"]
    for k in ("el_out", "er_out"):
        o = kw.get(k)
        if o is not None and (not o.is_contiguous() or o.numel() != n):
            raise ValueError(f"{k} must be a contiguous float32 CUDA tensor of n_dst elements")
    keep = _desc_vectors(info, op, F, kw)
    d = _desc(op, X, Y, F, ldx, ldy, **kw)
    sh = _stream(stream, X.device)
    _check(_lib.tlp_aggregate(g, ctypes.byref(d), sh), "tlp_aggregate")
    _keep_alive(sh, *keep)
    return Y


def tlp_sage_aggregate(g, X, include_self=False, Y=None, F=None, stream=None, n_dst=None, info=None):
    """GraphSage mean over N(v) (or N(v) + v with include_self)."""
    info, X, F, ldx, Y, ldy = _fwd_args(g, X, Y, F, info)
    _check(_lib.tlp_sage_aggregate(g, _ptr(X), F, ldx, int(bool(include_self)), _ptr(Y), ldy,
                                   _stream(stream, X.device)), "tlp_sage_aggregate")
    return Y


def tlp_gat_mh_aggregate(g, X, el, er, heads, slope=0.2, Y=None, F=None, stream=None, n_dst=None,
                         info=None):
    """Multi-head GAT; el: [n_src, heads], er: [n_dst (+row_offset), heads] CUDA fp32."""
    info, X, F, ldx, Y, ldy = _fwd_args(g, X, Y, F, info)
    el, er = _gat_vecs(info, el, er, int(heads))
    sh = _stream(stream, X.device)
    _check(_lib.tlp_gat_mh_aggregate(g, _ptr(X), int(heads), F, ldx, _ptr(el), _ptr(er),
                                     float(slope), _ptr(Y), ldy, sh), "tlp_gat_mh_aggregate")
    _keep_alive(sh, el, er)
    return Y


def _bwd_args(g, dY, dX, F, info):
    info = _info(g, info)
    dY, F, lddy = _feat(dY, F)
    _need_rows(dY, info["n_dst"], "dY")
    if dX is not None:
        _need_rows(_feat(dX, F)[0], info["n_src"], "dX")
    dX, F, lddx = _out(dX, info["n_src"], F, dY)
    return info, dY, F, lddy, dX, lddx


def tlp_gcn_backward(g, dY, norm="both", dX=None, F=None, stream=None, n_src=None, info=None):
    """dX = M^T dY for the GCN operator of the given norm (needs the transpose)."""
    info, dY, F, lddy, dX, lddx = _bwd_args(g, dY, dX, F, info)
    nm = NORMS[norm] if isinstance(norm, str) else int(norm)
    _check(_lib.tlp_gcn_backward(g, _ptr(dY), F, lddy, nm, _ptr(dX), lddx, _stream(stream, dY.device)),
           "tlp_gcn_backward")
    return dX


def tlp_gin_backward(g, dY, eps=0.0, dX=None, F=None, stream=None, n_src=None, info=None):
    info, dY, F, lddy, dX, lddx = _bwd_args(g, dY, dX, F, info)
    _check(_lib.tlp_gin_backward(g, _ptr(dY), F, lddy, float(eps), _ptr(dX), lddx,
                                 _stream(stream, dY.device)), "tlp_gin_backward")
    return dX


def tlp_gat_backward(g, X, el, er, slope, Y, dY, dX=None, F=None, stream=None, info=None):
    """Single-head GAT backward: returns (dX [n_src, F], del [n_src], der [n_dst]).
    Y is the forward output of tlp_gat_aggregate for the same X, el, er."""
    torch = _torch()
    info, dY, F, lddy, dX, lddx = _bwd_args(g, dY, dX, F, info)
    X, _, ldx = _feat(X, F)
    _need_rows(X, info["n_src"], "X")
    Y, _, ldy = _feat(Y, F)
    _need_rows(Y, info["n_dst"], "Y")
    el, er = _gat_vecs(info, el, er)
    dl = torch.empty(info["n_src"], dtype=torch.float32, device=dY.device)
    dr = torch.empty(info["n_dst"], dtype=torch.float32, device=dY.device)
    sh = _stream(stream, dY.device)
    _check(_lib.tlp_gat_backward(g, _ptr(X), F, ldx, _ptr(el), _ptr(er), float(slope), _ptr(Y), ldy,
                                 _ptr(dY), lddy, _ptr(dX), lddx, _ptr(dl), _ptr(dr), sh),
           "tlp_gat_backward")
    _keep_alive(sh, el, er)
    return dX, dl, dr


# -------------------------------------------------------------- multi-GPU ----

def tlp_partition_rows(rowptr, parts):
    rp = np.ascontiguousarray(rowptr, dtype=np.int64)
    b = np.empty(int(parts) + 1, np.int64)
    _check(_lib.tlp_partition_rows(_ptr(rp), rp.shape[0] - 1, int(parts), _ptr(b)),
           "tlp_partition_rows")
    return b


def tlp_comm_get_unique_id():
    buf = (ctypes.c_uint8 * 128)()
    _check(_lib.tlp_comm_get_unique_id(buf), "tlp_comm_get_unique_id")
    return bytes(buf)


def tlp_comm_create(uid, world, rank):
    if len(uid) != 128:
        raise ValueError("unique id must be 128 bytes")
    buf = (ctypes.c_uint8 * 128).from_buffer_copy(uid)
    out = _P()
    _check(_lib.tlp_comm_create(buf, int(world), int(rank), ctypes.byref(out)), "tlp_comm_create")
    return out.value


def tlp_comm_destroy(c):
    _check(_lib.tlp_comm_destroy(c), "tlp_comm_destroy")


def comm_from_torch(group=None):
    """NCCL communicator for the current torch.distributed world; torch only
    broadcasts the 128-byte id (rank 0 -> all)."""
    torch = _torch()
    import torch.distributed as dist
    rank, world = dist.get_rank(group), dist.get_world_size(group)
    obj = [tlp_comm_get_unique_id() if rank == 0 else None]
    dist.broadcast_object_list(obj, src=0, group=group)
    return tlp_comm_create(obj[0], world, rank)


def tlp_dist_graph_create(comm, rowptr, colidx, edge_weight=None, opts=None, stream=None):
    rowptr = _as_index(rowptr, np.int64)
    colidx = _as_index(colidx, np.int32)
    ew = None if edge_weight is None else _as_index(edge_weight, np.float32)
    n = int(rowptr.shape[0]) - 1
    out = _P()
    o = None
    if opts:
        o = tlp_create_opts(int(opts.get("hub_threshold", 0)), int(opts.get("hub_chunk", 0)),
                            int(opts.get("unit_edges", 0)))
    st = _lib.tlp_dist_graph_create(comm, n, int(colidx.shape[0]), _ptr(rowptr), _ptr(colidx),
                                    _ptr(ew), ctypes.byref(o) if o else None, _stream(stream),
                                    ctypes.byref(out))
    _check(st, "tlp_dist_graph_create")
    return out.value


def tlp_dist_bounds(g, world):
    b = np.empty(int(world) + 1, np.int64)
    _check(_lib.tlp_dist_bounds(g, _ptr(b)), "tlp_dist_bounds")
    return b


def _dist_args(g, X_full, Y_full, F):
    """X_full [n x ldx] replicated, Y_full [n x ldy] (n = the global row count)."""
    info = tlp_graph_info_get(g)
    n = info["n_src"]
    X, F, ldx = _feat(X_full, F)
    _need_rows(X, n, "X_full")
    Y, _, ldy = _feat(Y_full, F)
    _need_rows(Y, n, "Y_full")
    return info, n, X, F, ldx, Y, ldy


def tlp_dist_allgather_rows(g, comm, Y_full, stream=None):
    Y, F, ldy = _feat(Y_full, None)
    _need_rows(Y, tlp_graph_info_get(g)["n_src"], "Y_full")
    _check(_lib.tlp_dist_allgather_rows(g, comm, _ptr(Y), ldy, _stream(stream, Y.device)),
           "tlp_dist_allgather_rows")
    return Y_full


def tlp_dist_gcn_aggregate(g, comm, X_full, Y_full, norm="both", F=None, stream=None):
    info, n, X, F, ldx, Y, ldy = _dist_args(g, X_full, Y_full, F)
    nm = NORMS[norm] if isinstance(norm, str) else int(norm)
    _check(_lib.tlp_dist_gcn_aggregate(g, comm, _ptr(X), F, ldx, nm, _ptr(Y), ldy,
                                       _stream(stream, X.device)), "tlp_dist_gcn_aggregate")
    return Y_full


def tlp_dist_gin_aggregate(g, comm, X_full, Y_full, eps=0.0, F=None, stream=None):
    info, n, X, F, ldx, Y, ldy = _dist_args(g, X_full, Y_full, F)
    _check(_lib.tlp_dist_gin_aggregate(g, comm, _ptr(X), F, ldx, float(eps), _ptr(Y), ldy,
                                       _stream(stream, X.device)), "tlp_dist_gin_aggregate")
    return Y_full


def tlp_dist_gat_aggregate(g, comm, X_full, Y_full, el, er, slope=0.2, F=None, stream=None):
    info, n, X, F, ldx, Y, ldy = _dist_args(g, X_full, Y_full, F)
    el = _vec_cuda(el, "el", n)
    er = _vec_cuda(er, "er", n)
    sh = _stream(stream, X.device)
    _check(_lib.tlp_dist_gat_aggregate(g, comm, _ptr(X), F, ldx, _ptr(el), _ptr(er), float(slope),
                                       _ptr(Y), ldy, sh), "tlp_dist_gat_aggregate")
    _keep_alive(sh, el, er)
    return Y_full


def tlp_comm_async_error(comm):
    """The communicator's asynchronous NCCL state (0 = ncclSuccess); raises on an error."""
    r = _I()
    _check(_lib.tlp_comm_async_error(comm, ctypes.byref(r)), "tlp_comm_async_error")
    return r.value


def tlp_comm_abort(comm):
    _check(_lib.tlp_comm_abort(comm), "tlp_comm_abort")


def tlp_comm_wait(comm, stream=None, timeout_s=0.0):
    """Drain `stream` while polling NCCL's async error state; abort the
    communicator on an error or after timeout_s seconds (TlpError)."""
    _check(_lib.tlp_comm_wait(comm, _stream(stream), float(timeout_s)), "tlp_comm_wait")


class _CudaArray:
    """Zero-copy torch view of library-owned device memory (CUDA array interface)."""

    def __init__(self, ptr, shape):
        self.__cuda_array_interface__ = {"shape": tuple(shape), "typestr": "<f4",
                                         "data": (int(ptr), False), "version": 3, "strides": None}


def tlp_comm_alloc_symmetric(comm, rows, ld):
    """Collective: a [rows x ld] fp32 buffer on every rank, peer-mapped over NVLink.
    Returns (tensor view, raw pointer); free with tlp_comm_free_symmetric."""
    torch = _torch()
    out = _P()
    _check(_lib.tlp_comm_alloc_symmetric(comm, int(rows) * int(ld) * 4, ctypes.byref(out)),
           "tlp_comm_alloc_symmetric")
    t = torch.as_tensor(_CudaArray(out.value, (int(rows), int(ld))), device="cuda")
    return t, out.value


SYM_KINDS = {0: "ipc", 1: "nccl_window", 2: "nccl_window_multicast"}


def tlp_comm_symmetric_kind(comm, ptr):
    """'ipc', 'nccl_window' or 'nccl_window_multicast' (NVLS)."""
    k = _I()
    _check(_lib.tlp_comm_symmetric_kind(comm, ptr, ctypes.byref(k)), "tlp_comm_symmetric_kind")
    return SYM_KINDS.get(k.value, k.value)


def tlp_comm_free_symmetric(comm, ptr):
    _check(_lib.tlp_comm_free_symmetric(comm, ptr), "tlp_comm_free_symmetric")


def tlp_dist_aggregate_fused(g, comm, op, X_full, Y_sym, F=None, stream=None, **kw):
    """NEXT-2: one kernel computes this rank's rows and stores them into Y_full on
    every rank (Y_sym from tlp_comm_alloc_symmetric)."""
    info, n, X, F, ldx, Y, ldy = _dist_args(g, X_full, Y_sym, F)
    keep = _desc_vectors(info, op, F, kw, n_rows_global=n)
    d = _desc(op, X, Y, F, ldx, ldy, **kw)
    sh = _stream(stream, X.device)
    _check(_lib.tlp_dist_aggregate_fused(g, comm, ctypes.byref(d), sh), "tlp_dist_aggregate_fused")
    _keep_alive(sh, *keep)
    return Y_sym


def tlp_debug_multi_store(g, op, X, dests, F=None, stream=None, **kw):
    """Test hook: store the aggregation's output rows into every tensor of `dests`."""
    info = tlp_graph_info_get(g)
    X, F, ldx = _feat(X, F)
    _need_rows(X, info["n_src"], "X")
    D0, _, ldy = _feat(dests[0], F)
    for t in dests:
        _need_rows(_feat(t, F)[0], info["row_offset"] + info["n_dst"], "dest")
    keep = _desc_vectors(info, op, F, kw)
    d = _desc(op, X, D0, F, ldx, ldy, **kw)
    arr = (ctypes.c_void_p * len(dests))(*[t.data_ptr() for t in dests])
    _check(_lib.tlp_debug_multi_store(g, ctypes.byref(d), arr, len(dests), _stream(stream, X.device)),
           "tlp_debug_multi_store")
    del keep  # the call is synchronous
    return dests


def tlp_dist_aggregate(g, comm, op, X_full, Y_full, F=None, stream=None, **kw):
    info, n, X, F, ldx, Y, ldy = _dist_args(g, X_full, Y_full, F)
    keep = _desc_vectors(info, op, F, kw, n_rows_global=n)
    d = _desc(op, X, Y, F, ldx, ldy, **kw)
    sh = _stream(stream, X.device)
    _check(_lib.tlp_dist_aggregate(g, comm, ctypes.byref(d), sh), "tlp_dist_aggregate")
    _keep_alive(sh, *keep)
    return Y_full


def tlp_dist_sage_aggregate(g, comm, X_full, Y_full, include_self=False, F=None, stream=None):
    info, n, X, F, ldx, Y, ldy = _dist_args(g, X_full, Y_full, F)
    _check(_lib.tlp_dist_sage_aggregate(g, comm, _ptr(X), F, ldx, int(bool(include_self)), _ptr(Y),
                                        ldy, _stream(stream, X.device)), "tlp_dist_sage_aggregate")
    return Y_full


def tlp_dist_gat_mh_aggregate(g, comm, X_full, Y_full, el, er, heads, slope=0.2, F=None,
                              stream=None):
    info, n, X, F, ldx, Y, ldy = _dist_args(g, X_full, Y_full, F)
    el = _vec_cuda(el, "el", n * int(heads))
    er = _vec_cuda(er, "er", n * int(heads))
    sh = _stream(stream, X.device)
    _check(_lib.tlp_dist_gat_mh_aggregate(g, comm, _ptr(X), int(heads), F, ldx, _ptr(el), _ptr(er),
                                          float(slope), _ptr(Y), ldy, sh),
           "tlp_dist_gat_mh_aggregate")
    _keep_alive(sh, el, er)
    return Y_full


# ------------------------------------------------------------ convenience ---

class Graph:
    """Owning wrapper of a tlp_graph handle."""

    def __init__(self, rowptr, colidx, n_src=None, edge_weight=None, opts=None, stream=None,
                 handle=None):
        self.handle = handle if handle is not None else tlp_graph_create(
            rowptr, colidx, n_src=n_src, edge_weight=edge_weight, opts=opts, stream=stream)
        self.info = tlp_graph_info_get(self.handle)

    @classmethod
    def dist(cls, comm, rowptr, colidx, edge_weight=None, opts=None, stream=None):
        h = tlp_dist_graph_create(comm, rowptr, colidx, edge_weight=edge_weight, opts=opts,
                                  stream=stream)
        return cls(None, None, handle=h)

    @property
    def n_dst(self):
        return self.info["n_dst"]

    def gcn(self, X, norm="both", Y=None, F=None, stream=None):
        return tlp_gcn_aggregate(self.handle, X, norm, Y, F, stream, info=self.info)

    def gin(self, X, eps=0.0, Y=None, F=None, stream=None):
        return tlp_gin_aggregate(self.handle, X, eps, Y, F, stream, info=self.info)

    def gat(self, X, el, er, slope=0.2, Y=None, F=None, stream=None):
        return tlp_gat_aggregate(self.handle, X, el, er, slope, Y, F, stream, info=self.info)

    def sage(self, X, include_self=False, Y=None, F=None, stream=None):
        return tlp_sage_aggregate(self.handle, X, include_self, Y, F, stream, info=self.info)

    def gat_mh(self, X, el, er, heads, slope=0.2, Y=None, F=None, stream=None):
        return tlp_gat_mh_aggregate(self.handle, X, el, er, heads, slope, Y, F, stream,
                                    info=self.info)

    def aggregate(self, op, X, Y=None, F=None, stream=None, **kw):
        return tlp_aggregate(self.handle, op, X, Y, F, stream, info=self.info, **kw)

    def build_transpose(self, stream=None):
        tlp_graph_build_transpose(self.handle, stream)

    def gcn_backward(self, dY, norm="both", dX=None, F=None, stream=None):
        return tlp_gcn_backward(self.handle, dY, norm, dX, F, stream, info=self.info)

    def gin_backward(self, dY, eps=0.0, dX=None, F=None, stream=None):
        return tlp_gin_backward(self.handle, dY, eps, dX, F, stream, info=self.info)

    def gat_backward(self, X, el, er, slope, Y, dY, dX=None, F=None, stream=None):
        return tlp_gat_backward(self.handle, X, el, er, slope, Y, dY, dX, F, stream, info=self.info)

    def degrees(self):
        return tlp_graph_degrees(self.handle)

    def plan(self):
        return tlp_graph_plan(self.handle)

    def set_schedule(self, sched="dynamic", warps_per_cta=0, step=0):
        tlp_graph_set_schedule(self.handle, sched, warps_per_cta, step)

    def close(self):
        if self.handle:
            tlp_graph_destroy(self.handle)
            self.handle = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass

    def __enter__(self):
        return self

    def __exit__(self, *a):
        self.close()

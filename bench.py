#!/usr/bin/env python
"""Benchmark of the TLPGNN aggregation hot path on B200 (driver contract).

A step = one pass of the whole hot path over the Reddit-shaped graph
(BASELINE.json configs[2]: N = 232,965, E = 114,615,892, F = 602, ld = 604):
GCN (BOTH norm) + GIN (eps 0.1) + GAT (slope 0.2), each ONE kernel launch of
libtlp through the C ABI.  The graph handle (ingest/validate/degrees/plan,
SURVEY 8(a) a1-a3) is created once before the timed region, as the structure
is static across layers; its create time is reported separately.

value = gather-model bytes of the step / device time (GB/s):
  GCN per edge 4F + 4 (colidx) + 4 (c_out[u]); per row 4F (Y) + 8 (rowptr)
  GIN per edge 4F + 4;                          per row 8F + 8 (self + Y)
  GAT per edge 4F + 4 + 4 (el[u]);              per row 4F + 12 (Y, rowptr, er)
N > 1 (torchrun): destination rows split by edge count, X replicated, every
aggregation followed by the all-gather of Y rows (tlp_dist_*); total work is
fixed ("strong" scaling); time = max over ranks.

--impl reference: the fp64 oracle (oracle/, single-threaded C) timed on the
host cores on a bounded row sample of the same workload -- the paper ships no
code, so the oracle is this tier's reference arm.
"""
from __future__ import annotations

import argparse
import json
import os
import statistics
import subprocess
import sys
import threading
import time

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

import numpy as np  # noqa: E402

METRIC = "GCN/GAT aggregation ms & HBM GB/s vs 8 TB/s, Reddit-shaped, 1/2/4/8 B200"
NOMINAL_HBM_GBS = 8000.0
FALLBACK_HBM_GBS = 6650.0  # B200_PROFILING.md fallback, used only without MEASURED_PEAKS.json
OPS = ("gcn", "gin", "gat")
# "gcn2": two GCN(BOTH) layers, Y1 = A X, Y2 = A Y1 (the R-MAT config; X.W is out of scope)


# ------------------------------------------------------------------ bytes --


def _sig(x, digits=5):
    """x rounded to `digits` significant digits (small-graph steps are ~0.02 ms)."""
    if not x:
        return x
    import math
    return round(x, max(0, digits - 1 - int(math.floor(math.log10(abs(x))))))

def gather_bytes(op, n_rows, n_edges, F):
    """Algorithmic (gather-model) bytes of one aggregation."""
    if op == "gcn":
        return n_edges * (4 * F + 8) + n_rows * (4 * F + 8)
    if op == "gin":
        return n_edges * (4 * F + 4) + n_rows * (8 * F + 8)
    if op == "gat":
        return n_edges * (4 * F + 8) + n_rows * (4 * F + 12)
    if op == "gcn2":
        return 2 * gather_bytes("gcn", n_rows, n_edges, F)
    if op == "gcn_bwd":  # dX = M^T dY on the transposed CSR: same byte model as GCN
        return gather_bytes("gcn", n_rows, n_edges, F)
    if op == "gat_bwd":
        # GAT backward (tlp_gat_backward): per edge one dY row (4F) on the
        # transposed CSR, plus the scalar edge streams of its four passes
        # (colidx/el 8, colidx/vstat/dot 24, colidx/vstat/dot/dt 28, tpos/dt 8);
        # per row dY.Y (8F), X[u] and dX[u] (8F) and ~60 B of row scalars
        return n_edges * (4 * F + 68) + n_rows * (16 * F + 60)
    if op == "sage":  # mean over N(v)+v: per edge 4F + 4; per row self + Y + rowptr
        return n_edges * (4 * F + 4) + n_rows * (8 * F + 8)
    if op.startswith("gat") and op[3:].isdigit():  # H heads: el/er per head
        H = int(op[3:])
        return n_edges * (4 * F + 4 + 4 * H) + n_rows * (4 * F + 8 + 4 * H)
    raise ValueError(op)


def l2_gather_ceiling(table_bytes, iters=600):
    """In-run L2 random-row gather ceiling (bench_probe/l2_ceiling.cu, built by
    __graft_entry__.build()): GB/s of 256-byte random-row gathers from an
    L2-resident table of `table_bytes` (one panel-major strip block), or None."""
    import ctypes
    p = os.path.join(ROOT, "bench_probe", "libl2c.so")
    if not os.path.exists(p):
        return None
    lib = ctypes.CDLL(p)
    lib.l2c_run.argtypes = [ctypes.c_int64, ctypes.c_int, ctypes.POINTER(ctypes.c_float),
                            ctypes.POINTER(ctypes.c_double)]
    ms, by = ctypes.c_float(), ctypes.c_double()
    if lib.l2c_run(int(table_bytes), int(iters), ctypes.byref(ms), ctypes.byref(by)) != 0:
        return None
    return {"GBs": round(by.value / (ms.value * 1e-3) / 1e9, 1), "ms": round(ms.value, 3),
            "table_MB": round(table_bytes / 1e6, 1)}


def cpu_model():
    try:
        for line in open("/proc/cpuinfo"):
            if line.startswith("model name"):
                return line.split(":", 1)[1].strip()
    except OSError:
        pass
    return None


def peak_hbm():
    p = os.path.join(ROOT, "MEASURED_PEAKS.json")
    try:
        with open(p) as f:
            v = float(json.load(f)["hbm_gbs"])
        return v, "measured (MEASURED_PEAKS.json hbm_gbs)"
    except Exception:
        return FALLBACK_HBM_GBS, "fallback (B200_PROFILING.md)"


def load_traffic(workload):
    """DRAM bytes per launch from the committed ncu --set full summary."""
    p = os.path.join(ROOT, "profiles", "ncu_traffic.json")
    try:
        with open(p) as f:
            d = json.load(f).get(workload, {})
        # R-MAT's timed op is two GCN layers of the same shape: two launches
        # of the captured per-layer kernel
        if workload == "rmat24" and "gcn" in d and "gcn2" not in d:
            d["gcn2"] = 2 * d["gcn"]
        return d
    except Exception:
        return {}


# ------------------------------------------------------------------ clocks --

class ClockSampler:
    """nvidia-smi clocks / throttle reasons sampled DURING the timed region."""
    Q = ("index,clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.active,"
         "clocks_event_reasons.hw_slowdown,clocks_event_reasons.hw_thermal_slowdown,"
         "clocks_event_reasons.sw_thermal_slowdown,clocks_event_reasons.sw_power_cap")

    def __init__(self, gpu_index, period_ms=None):
        self.gpu = gpu_index
        self.period = int(period_ms or os.environ.get("TLP_CLOCK_MS", "50"))
        self.proc = None
        self.lines = []
        self.stamps = []
        self.t0 = 0.0

    def __enter__(self):
        if self.period <= 0:
            return self
        try:
            self.proc = subprocess.Popen(
                ["nvidia-smi", "--query-gpu=" + self.Q, "--format=csv,noheader,nounits",
                 "-lms", str(self.period), "-i", str(self.gpu)],
                stdout=subprocess.PIPE, stderr=subprocess.DEVNULL, text=True)
            self.t = threading.Thread(target=self._read, daemon=True)
            self.t.start()
            # nvidia-smi takes a few hundred ms to emit its first sample: wait
            # for it, so the region that follows is sampled from its start
            t_wait = time.time() + 3.0
            while not self.lines and time.time() < t_wait:
                time.sleep(0.005)
            self.t0 = time.time()
        except Exception:
            self.proc = None
        return self

    def _read(self):
        for line in self.proc.stdout:
            self.stamps.append(time.time())
            self.lines.append(line.strip())

    def __exit__(self, *a):
        if self.proc:
            self.proc.terminate()
            try:
                self.proc.wait(timeout=5)
            except Exception:
                self.proc.kill()
            self.t.join(timeout=2)

    def summary(self):
        sm, mx, reasons = [], [], set()
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        stamps = self.stamps + [float("inf")] * (len(self.lines) - len(self.stamps))
        for ts, ln in zip(stamps, self.lines):
            if ts < self.t0:  # the warm-up sample taken before the region
                continue
            parts = [p.strip() for p in ln.split(",")]
            if len(parts) < 9:
                continue
            try:
                sm.append(float(parts[1]))
                mx.append(float(parts[2]))
            except ValueError:
                continue
            for nm, v in zip(names, parts[5:9]):
                if v.lower().startswith("active"):
                    reasons.add(nm)
        if not sm:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": [], "samples": 0}
        return {"sm_mhz": statistics.median(sm), "sm_max_mhz": max(mx),
                "reasons": sorted(reasons), "samples": len(sm)}


# ---------------------------------------------------------------- workload --

WORKLOADS = {
    "reddit": dict(graph="reddit", ops=OPS),
    "products": dict(graph="products", ops=("gat",)),
    # single-op Reddit workloads (kernel experiments)
    "reddit_gcn": dict(graph="reddit", ops=("gcn",)),
    "reddit_gin": dict(graph="reddit", ops=("gin",)),
    "reddit_gat": dict(graph="reddit", ops=("gat",)),
    # the paper's own measurement shape (F = 32; Table 5): context for
    # its V100 numbers, not a BASELINE.json config
    "reddit_f32": dict(graph="reddit", ops=OPS, F=32, ld=32,
                       paper_v100_ms={"gcn": 6.9, "gin": 7.3, "gat": 14.6},
                       paper_src="PAPER.md Table 5 P:1175, P:1189, P:1217 (V100 32 GB, F=32, mean of 10)"),
    "products_f32": dict(graph="products", ops=OPS, F=32, ld=32,
                         paper_v100_ms={"gcn": 16.1, "gin": 16.4, "gat": 28.4},
                         paper_src="PAPER.md Table 5 P:1179, P:1193, P:1221 (V100 32 GB, F=32, mean of 10)"),
    "pubmed": dict(graph="pubmed", ops=("gat",)),
    "cora": dict(graph="cora", ops=("gcn",)),
    "rmat24": dict(graph="rmat24", ops=("gcn2",)),
    # NEXT-1 rows: GraphSage mean (+self) and 4-head GAT
    "reddit_sage": dict(graph="reddit", ops=("sage",)),
    "products_gat4": dict(graph="products", ops=("gat4",)),
    # NEXT-4: the backward aggregation of a GCN(BOTH) layer
    "reddit_bwd": dict(graph="reddit", ops=("gcn_bwd",)),
    "reddit_gat_bwd": dict(graph="reddit", ops=("gat_bwd",)),
    "pubmed_gat_bwd": dict(graph="pubmed", ops=("gat_bwd",)),
}


def workload_desc(name, cfg, E):
    ops = "+".join({"gcn": "GCN(both)", "gin": "GIN(eps=0.1)", "gat": "GAT(slope=0.2)",
                    "gcn2": "2-layer GCN(both)", "sage": "GraphSage-mean(+self)",
                    "gat4": "4-head GAT(slope=0.2)",
                    "gcn_bwd": "GCN(both) backward dX = M^T dY",
                    "gat_bwd": "GAT(slope=0.2) backward (dX, del, der)"}[o] for o in WORKLOADS[name]["ops"])
    return f"{name}-shaped {ops}: N={cfg_n(cfg)} E={E} F={cfg['F']} ld={cfg['ld']}"


def cfg_n(cfg):
    return cfg["n"] if "n" in cfg else 1 << cfg["scale"]


def make_inputs(name, device):
    import synth
    w = WORKLOADS[name]
    cfg = synth.CONFIGS[w["graph"]]
    rp, ci = synth.dataset_graph(w["graph"], device=device)
    n = cfg_n(cfg)
    if "F" in w:  # feature width override (the paper's F = 32 shape)
        cfg = dict(cfg, F=w["F"], ld=w["ld"])
        X = synth.features(n, w["F"], w["ld"], seed=synth.FEATURE_SEED_BASE + synth.CONFIG_INDEX[w["graph"]])
    else:
        X = synth.dataset_features(w["graph"], n)
    H = max([int(o[3:]) for o in WORKLOADS[name]["ops"] if o.startswith("gat") and o[3:].isdigit()]
            or [1])
    el = synth.normal(n * H, 1000 + synth.CONFIG_INDEX[WORKLOADS[name]["graph"]])
    er = synth.normal(n * H, 2000 + synth.CONFIG_INDEX[WORKLOADS[name]["graph"]])
    return cfg, rp, ci, X, el, er


# --------------------------------------------------------------- our arm ----

def run_tlp(args):
    import torch
    import torch.distributed as dist
    import paper_conf_hpdc_fujh22_b200 as tlp
    import synth

    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    torch.cuda.set_device(local)
    dev = torch.device("cuda", local)
    # the dist path (NCCL comm + tlp_dist_*) also at world = 1 with --dist
    use_dist = world > 1 or args.dist
    if use_dist:
        # the driver counts ranks from NCCL's init log (read by NCCL at its
        # first communicator, i.e. before the process group comes up)
        os.environ.setdefault("NCCL_DEBUG", "INFO")
        os.environ.setdefault("NCCL_DEBUG_SUBSYS", "INIT")
        os.environ.setdefault("MASTER_ADDR", "127.0.0.1")
        os.environ.setdefault("MASTER_PORT", str(29500 + os.getpid() % 1000))
        dist.init_process_group("nccl", device_id=dev, rank=rank, world_size=world)
    name = args.workload
    ops = WORKLOADS[name]["ops"]
    cfg, rp, ci, Xh, elh, erh = make_inputs(name, dev)
    n, F, ld = cfg_n(cfg), cfg["F"], cfg["ld"]
    E = len(ci)
    stream = torch.cuda.current_stream(dev)

    rp_d = torch.from_numpy(rp).to(dev)
    ci_d = torch.from_numpy(ci).to(dev)
    comm = None
    if use_dist:
        comm = tlp.comm_from_torch()
    # first create of the process: includes loading the library's create
    # kernels (CUDA lazy module loading); then the warm create of the real
    # graph (SURVEY 8(a) a1 target: create < 1 % of one aggregation)
    t0 = time.perf_counter()
    tiny = tlp.Graph(torch.tensor([0, 1], device=dev), torch.tensor([0], dtype=torch.int32, device=dev))
    torch.cuda.synchronize()
    first_create_ms = (time.perf_counter() - t0) * 1e3
    tiny.close()

    def create():
        t0 = time.perf_counter()
        h = tlp.Graph.dist(comm, rp_d, ci_d) if use_dist else tlp.Graph(rp_d, ci_d)
        torch.cuda.synchronize()
        return h, (time.perf_counter() - t0) * 1e3

    # the first create of the full graph also pays the first large device
    # allocations of the process; the handle used below is a second create
    g, create_cold_ms = create()
    g.close()
    g, create_ms = create()
    if "gcn_bwd" in ops or "gat_bwd" in ops:
        g.build_transpose()
    info = g.info
    del ci_d
    X = torch.from_numpy(Xh).to(dev)
    el = torch.from_numpy(elh).to(dev)
    er = torch.from_numpy(erh).to(dev)
    sym_ptrs = []
    fused = use_dist and args.fused

    def out_buffer():
        if fused:  # NEXT-2: NVLink-mapped symmetric Y_full written by the kernel itself
            t_, p_ = tlp.tlp_comm_alloc_symmetric(comm, n, ld)
            sym_ptrs.append(p_)
            return t_
        return torch.empty((n, ld), dtype=torch.float32, device=dev)

    Y = {op: out_buffer() for op in ops}
    sym_kind = tlp.tlp_comm_symmetric_kind(comm, sym_ptrs[0]) if (fused and sym_ptrs) else None
    Y1 = out_buffer() if "gcn2" in ops else None

    def gcn_to(Xin, out):
        if fused:
            tlp.tlp_dist_aggregate_fused(g.handle, comm, "gcn", Xin, out, F=F, norm="both")
        elif use_dist:
            tlp.tlp_dist_gcn_aggregate(g.handle, comm, Xin, out, "both", F=F)
        else:
            g.gcn(Xin, "both", Y=out, F=F)

    def launch(op, Xin=X, elv=el, erv=er, Yo=Y):
        if op == "gcn2":  # layer 1, then layer 2 on its output (all-gather between in dist mode)
            gcn_to(Xin, Y1)
            gcn_to(Y1, Yo[op])
        elif op == "gcn":
            gcn_to(Xin, Yo[op])
        elif op == "gcn_bwd":
            g.gcn_backward(Xin, "both", dX=Yo[op], F=F)
        elif op == "gat_bwd":  # dY = Xin, forward output Yfwd (computed once below)
            g.gat_backward(X, elv, erv, synth.SLOPE, Yfwd, Xin, dX=Yo[op], F=F)
        elif fused:
            kw = dict(eps=synth.EPS, slope=synth.SLOPE, include_self=True)
            if op.startswith("gat"):
                kw.update(el=elv, er=erv, heads=int(op[3:]) if op[3:].isdigit() else 1)
            tlp.tlp_dist_aggregate_fused(g.handle, comm, "gat_mh" if op[3:].isdigit() else op,
                                         Xin, Yo[op], F=F, **kw)
        elif use_dist:
            if op == "gin":
                tlp.tlp_dist_gin_aggregate(g.handle, comm, Xin, Yo[op], synth.EPS, F=F)
            elif op == "sage":
                tlp.tlp_dist_sage_aggregate(g.handle, comm, Xin, Yo[op], True, F=F)
            elif op == "gat":
                tlp.tlp_dist_gat_aggregate(g.handle, comm, Xin, Yo[op], elv, erv, synth.SLOPE, F=F)
            else:
                tlp.tlp_dist_gat_mh_aggregate(g.handle, comm, Xin, Yo[op], elv, erv, int(op[3:]),
                                              synth.SLOPE, F=F)
        elif op == "gin":
            g.gin(Xin, synth.EPS, Y=Yo[op], F=F)
        elif op == "sage":
            g.sage(Xin, True, Y=Yo[op], F=F)
        elif op == "gat":
            g.gat(Xin, elv, erv, synth.SLOPE, Y=Yo[op], F=F)
        else:
            g.gat_mh(Xin, elv, erv, int(op[3:]), synth.SLOPE, Y=Yo[op], F=F)

    Yfwd = None
    if "gat_bwd" in ops:  # the forward output the backward takes (not timed)
        Yfwd = g.gat(X, el, er, synth.SLOPE, F=F)
    for _ in range(args.warmup):
        for op in ops:
            launch(op)
    torch.cuda.synchronize()

    # ---- device-resident timed region ----
    ev = {op: [] for op in ops}
    start, stop = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    graphs = None
    if args.cuda_graph:
        # launch-bound small graphs: one CUDA graph per op, replayed (no host gaps)
        graphs = {}
        side = torch.cuda.Stream(dev)
        side.wait_stream(stream)
        l_cap = tlp.tlp_graph_info_get(g.handle)["launches"]
        with torch.cuda.stream(side):
            for op in ops:
                cg = torch.cuda.CUDAGraph()
                with torch.cuda.graph(cg, stream=side):
                    launch(op)
                graphs[op] = cg
        # kernels per replayed step (counted by the library while capturing)
        graph_launches = tlp.tlp_graph_info_get(g.handle)["launches"] - l_cap
        stream.wait_stream(side)
        torch.cuda.synchronize()
        for op in ops:
            graphs[op].replay()
        torch.cuda.synchronize()
    if use_dist:
        dist.barrier()
    torch.cuda.synchronize()
    l_before = tlp.tlp_graph_info_get(g.handle)["launches"]
    with ClockSampler(local) as clk:
        # a one-op step is timed by the start / stop pair alone: per-launch
        # events would add host work between back-to-back launches of a
        # microsecond-scale kernel (Cora, Pubmed) and leave the GPU idle
        per_op_events = len(ops) > 1
        start.record(stream)
        for _ in range(args.steps):
            for op in ops:
                if per_op_events:
                    a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
                    a.record(stream)
                if graphs is not None:
                    for _r in range(args.graph_reps):
                        graphs[op].replay()
                else:
                    launch(op)
                if per_op_events:
                    b.record(stream)
                    ev[op].append((a, b))
        stop.record(stream)
        torch.cuda.synchronize()
    if use_dist:
        dist.barrier()
    # our kernels launched inside the timed region, as counted by the library
    if graphs is not None:
        n_launches = graph_launches * args.graph_reps * args.steps
    else:
        n_launches = tlp.tlp_graph_info_get(g.handle)["launches"] - l_before
    reps = args.graph_reps if graphs is not None else 1
    total_ms = start.elapsed_time(stop) / reps
    if per_op_events:
        op_ms = {op: [a.elapsed_time(b) / reps for a, b in ev[op]] for op in ops}
    else:  # one op: its time per launch is the step time
        op_ms = {op: [total_ms / args.steps] for op in ops}
    t = torch.tensor([total_ms], device=dev)
    if use_dist:
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
        for op in ops:
            tt = torch.tensor(op_ms[op], device=dev)
            dist.all_reduce(tt, op=dist.ReduceOp.MAX)
            op_ms[op] = tt.tolist()
    total_ms = float(t.item())
    ms_per_step = total_ms / args.steps
    step_bytes = sum(gather_bytes(op, n, E, F) for op in ops)
    value = step_bytes / (ms_per_step * 1e-3) / 1e9

    # ---- SURVEY 8(d) d3 extras: host wall time of one API call (launch
    # overhead, not synchronised) and, with --cold, each op with L2 flushed
    host_us = {}
    for op in ops:
        hs = []
        for _ in range(21):
            torch.cuda.synchronize()
            t_h = time.perf_counter()
            launch(op)
            hs.append((time.perf_counter() - t_h) * 1e6)
        host_us[op] = statistics.median(hs)
        torch.cuda.synchronize()
    cold_ms = {}
    if args.cold:
        flush = torch.empty(int(2.5 * 126e6) // 4, dtype=torch.float32, device=dev)  # > 2x L2
        for op in ops:
            vals = []
            for _ in range(max(3, min(args.steps, 10))):
                flush.zero_()
                a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
                a.record(stream)
                launch(op)
                b.record(stream)
                torch.cuda.synchronize()
                vals.append(a.elapsed_time(b))
            cold_ms[op] = statistics.median(vals)
        del flush

    # ---- end to end through the public API with host buffers ----
    e2e = None
    if not args.no_e2e:
        Xp = torch.from_numpy(Xh).pin_memory()
        elp, erp = torch.from_numpy(elh).pin_memory(), torch.from_numpy(erh).pin_memory()
        # every rank uploads its (replicated) inputs; rank 0 reads the result back
        read_back = rank == 0
        Yp = {op: torch.empty((n, ld), dtype=torch.float32).pin_memory() for op in ops} if read_back else {}
        # Pipelined like a real caller: X/el/er double-buffered on the device,
        # uploads on one copy stream overlap the previous step's aggregations,
        # each Y is read back on a second copy stream while the next op runs.
        Xd = [X, torch.empty_like(X)]
        eld, erd = [el, torch.empty_like(el)], [er, torch.empty_like(er)]
        Yd = [Y, {op: out_buffer() for op in ops}]
        s_h2d, s_d2h = torch.cuda.Stream(dev), torch.cuda.Stream(dev)
        comp_done, d2h_done = [None, None], [{}, {}]
        if use_dist:
            dist.barrier()
        torch.cuda.synchronize()
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        a.record(stream)
        s_h2d.wait_event(a)
        s_d2h.wait_event(a)
        for i in range(args.steps):
            k = i % 2
            with torch.cuda.stream(s_h2d):
                if comp_done[k] is not None:
                    s_h2d.wait_event(comp_done[k])
                Xd[k].copy_(Xp, non_blocking=True)
                eld[k].copy_(elp, non_blocking=True)
                erd[k].copy_(erp, non_blocking=True)
                up = torch.cuda.Event()
                up.record(s_h2d)
            stream.wait_event(up)
            for op in ops:
                if op in d2h_done[k]:
                    stream.wait_event(d2h_done[k][op])
                launch(op, Xd[k], eld[k], erd[k], Yd[k])
                if read_back:
                    ready = torch.cuda.Event()
                    ready.record(stream)
                    with torch.cuda.stream(s_d2h):
                        s_d2h.wait_event(ready)
                        Yp[op].copy_(Yd[k][op], non_blocking=True)
                        dn = torch.cuda.Event()
                        dn.record(s_d2h)
                        d2h_done[k][op] = dn
            cd = torch.cuda.Event()
            cd.record(stream)
            comp_done[k] = cd
        stream.wait_stream(s_h2d)
        stream.wait_stream(s_d2h)
        b.record(stream)
        torch.cuda.synchronize()
        last = Yd[(args.steps - 1) % 2]
        te = torch.tensor([a.elapsed_time(b)], device=dev)
        if use_dist:
            dist.all_reduce(te, op=dist.ReduceOp.MAX)
        e2e_ms = float(te.item()) / args.steps
        h2d = Xp.numel() * 4 + elp.numel() * 4 + erp.numel() * 4
        d2h = sum(Yp[op].numel() * 4 for op in ops) if read_back else 0
        e2e = {"value": round(step_bytes / (e2e_ms * 1e-3) / 1e9, 2), "unit": "GB/s",
               "ms_per_step": _sig(e2e_ms), "h2d_bytes_per_step": int(h2d),
               "d2h_bytes_per_step": int(d2h),
               "note": "per step: pinned host X/el/er -> device (every rank), the step's "
                       "aggregations, every Y -> pinned host (rank 0); copies pipelined on two "
                       "streams against the aggregations (double-buffered); max over ranks"}
        # parity spot check of the end-to-end outputs (device copy vs host copy)
        for op in Yp:
            assert torch.equal(Yp[op][:64].to(dev), last[op][:64])

    # ---- dist: the local aggregation and the all-gather timed separately ----
    dist_split = None
    if use_dist and not fused and graphs is None and all(o in ("gcn", "gin", "gat", "sage") for o in ops):
        b = tlp.tlp_dist_bounds(g.handle, world)
        lo, hi = int(b[rank]), int(b[rank + 1])
        comp = {op: [] for op in ops}
        gath = {op: [] for op in ops}
        dist.barrier()
        torch.cuda.synchronize()
        for _ in range(max(3, min(args.steps, 10))):
            for op in ops:
                ys = Y[op][lo:hi]
                a1, a2, a3 = (torch.cuda.Event(enable_timing=True) for _ in range(3))
                a1.record(stream)
                if op in ("gcn", "gcn2"):
                    g.gcn(X, "both", Y=ys, F=F)
                elif op == "gin":
                    g.gin(X, synth.EPS, Y=ys, F=F)
                elif op == "sage":
                    g.sage(X, True, Y=ys, F=F)
                else:
                    g.gat(X, el, er, synth.SLOPE, Y=ys, F=F)
                a2.record(stream)
                tlp.tlp_dist_allgather_rows(g.handle, comm, Y[op], stream=stream)
                a3.record(stream)
                comp[op].append((a1, a2))
                gath[op].append((a2, a3))
        torch.cuda.synchronize()
        dist_split = {}
        for op in ops:
            tc = torch.tensor([statistics.median([x.elapsed_time(y) for x, y in comp[op]]),
                               statistics.median([x.elapsed_time(y) for x, y in gath[op]])], device=dev)
            dist.all_reduce(tc, op=dist.ReduceOp.MAX)
            ybytes = n * ld * 4
            dist_split[op] = {"compute_ms": round(float(tc[0]), 4), "allgather_ms": round(float(tc[1]), 4),
                              "allgather_bytes": int(ybytes),
                              "allgather_busbw_GBs": round(ybytes * (world - 1) / world
                                                           / (float(tc[1]) * 1e-3) / 1e9, 1)}

    # ---- roofline of the dominant kernel ----
    peak, peak_src = peak_hbm()
    per_op = {}
    for op in ops:
        ms = statistics.mean(op_ms[op])
        by = gather_bytes(op, n, E, F)
        srt = sorted(op_ms[op])
        per_op[op] = {"ms_mean": _sig(ms), "ms_median": _sig(statistics.median(op_ms[op])),
                      "ms_min": _sig(srt[0]),
                      "ms_p90": _sig(srt[min(len(srt) - 1, int(0.9 * len(srt)))]),
                      "host_call_us": round(host_us[op], 1),
                      "gather_bytes": int(by), "gather_GBs": round(by / (ms * 1e-3) / 1e9, 1),
                      "frac_of_8TBs": round(by / (ms * 1e-3) / 1e9 / NOMINAL_HBM_GBS, 4),
                      "edges_x_features_per_s": float(E * F / (ms * 1e-3))}
        if op in cold_ms:
            per_op[op]["ms_cold_l2_flushed"] = round(cold_ms[op], 4)
    dom = max(ops, key=lambda o: per_op[o]["ms_mean"])
    traffic = load_traffic(name).get(dom)
    achieved = per_op[dom]["gather_GBs"]
    # L2-panel mode (X larger than L2, a 64-column strip block fits): the
    # gathered rows are L2 hits, so the bound is the L2 random-row gather rate,
    # measured in this run by the probe (same clocks, same box)
    panel = n * ld * 4 > 0.6 * 126e6 and n * 256 <= 0.6 * 126e6 and F > 64
    # hub-free graphs whose X fits in L2 run the short-row kernel (tlp_k_rows.cu)
    kname = "k_rows" if (info["n_hubs"] == 0 and n * ld * 4 <= 0.6 * 126e6) else "k_agg"
    roofline = {"kernel": f"{kname} ({dom})", "achieved": achieved, "unit": "GB/s",
                "bytes_per_launch": per_op[dom]["gather_bytes"],
                "bytes_model": "gather model (SURVEY 8(d) d2): per edge 4F + 4 colidx + 4 coef/el; "
                               "per row Y, rowptr (+self/er); time = the op's mean CUDA-event "
                               "duration over the timed region (all of its launches; a one-op "
                               "step: the step time)",
                "traffic": traffic,
                "traffic_source": "profiles/ncu_traffic.json (dram__bytes_read.sum + "
                                  "dram__bytes_write.sum per launch, ncu --set full of this round's kernels)"}
    probe = None
    if panel and rank == 0:
        # probe runs for ~0.4 s so the clock sampler sees them; the best run is the ceiling
        runs = []
        with ClockSampler(local) as pclk:
            t_end = time.time() + 0.4  # >= ~8 clock samples
            while (time.time() < t_end or len(runs) < 30) and len(runs) < 2000:
                r_ = l2_gather_ceiling(n * 256)
                if not r_:
                    break
                runs.append(r_)
        if runs:
            probe = max(runs, key=lambda r_: r_["GBs"])
            probe["median_GBs"] = round(statistics.median(r_["GBs"] for r_ in runs), 1)
            probe["runs"] = len(runs)
            probe["clocks"] = pclk.summary()
    if probe:
        roofline.update({"bound": "l2", "peak": probe["GBs"], "frac": round(achieved / probe["GBs"], 4),
                         "peak_source": "measured in this run: bench_probe/l2_ceiling.cu, random "
                                        "256-byte rows of a %.0f MB L2-resident table (one strip "
                                        "block), persistent grid at the kernel's occupancy" % probe["table_MB"],
                         "probe": probe})
    else:
        roofline.update({"bound": "hbm", "peak": peak, "frac": round(achieved / peak, 4),
                         "peak_source": peak_src})
        if achieved > peak:
            roofline["note"] = ("frac > 1: the gather model counts one source-row read per edge, but "
                                "rows of high out-degree sources are re-read from L2 (hot-source "
                                "L2 policy), so the kernel moves fewer DRAM bytes than the model; "
                                "roofline.hbm is the DRAM-measured rate")
    if traffic:
        # DRAM bytes per launch over this run's launch time: the HBM rate
        roofline["hbm"] = {"achieved": round(traffic / (per_op[dom]["ms_mean"] * 1e-3) / 1e9, 1),
                           "peak": peak, "peak_source": peak_src, "unit": "GB/s"}
        roofline["hbm"]["frac"] = round(roofline["hbm"]["achieved"] / peak, 4)

    result = {
        "metric": METRIC, "value": round(value, 2), "unit": "GB/s", "n_gpus": world,
        "steps": args.steps, "warmup": args.warmup, "ms_per_step": _sig(ms_per_step),
        "higher_is_better": True, "scaling": "strong", "vs_baseline": None, "dtype": "f32",
        "data": "synthetic",
        "config": {"workload": workload_desc(name, cfg, E),
                   "graph": ("R-MAT G2 (0.57,0.19,0.19,0.05), seed %d" if name == "rmat24"
                             else "Chung-Lu G1 (SURVEY 8(d) d1), seed %d") % cfg["seed"],
                   "l2": ("inputs larger than L2 (X = %.0f MB, colidx = %.0f MB vs 126 MB L2); no flush"
                          % (n * ld * 4 / 1e6, E * 4 / 1e6)) if n * ld * 4 > 126e6 else
                         ("X = %.0f MB fits L2 (warm between reps); colidx = %.0f MB streams from HBM; "
                          "--cold adds L2-flushed times" % (n * ld * 4 / 1e6, E * 4 / 1e6)),
                   "parallelism": ("rows%d (edge-balanced row ranges, X replicated, %s)" % (
                       world, "fused peer-store all-gather (NEXT-2)" if fused else
                       "grouped-broadcast all-gather of Y")) if use_dist else "single",
                   "frac_of_8TBs": round(value / NOMINAL_HBM_GBS, 4),
                   "value_kind": "gather-model (logical) bytes of the step / device time: every edge "
                                 "counts one source-row read (SURVEY 8(d) d2); in L2-panel mode most of "
                                 "them are L2 hits, so it can exceed the HBM peak -- roofline.hbm holds "
                                 "the DRAM rate"},
        "ops": per_op, "create_ms": round(create_ms, 2),
        "create_cold_ms": round(create_cold_ms, 1), "create_first_tiny_ms": round(first_create_ms, 1),
        "plan": {k: info[k] for k in ("n_hubs", "n_hub_chunks", "n_units", "n_tasks",
                                      "hub_threshold", "hub_chunk", "max_in_degree")},
        "roofline": roofline,
        "gpu_launches": int(n_launches),
        "clocks": clk.summary(), "e2e": e2e,
    }
    if dist_split:
        result["dist"] = dist_split
    if sym_kind:
        result["config"]["symmetric_buffer"] = sym_kind
    w = WORKLOADS[name]
    if "paper_v100_ms" in w:
        # context only (another GPU, the paper's own F = 32 measurement)
        result["paper_context"] = {
            "v100_ms": w["paper_v100_ms"], "source": w["paper_src"],
            "b200_over_v100": {o: round(w["paper_v100_ms"][o] / per_op[o]["ms_mean"], 2)
                               for o in ops if o in w["paper_v100_ms"]}}
    if use_dist:
        result["gpu_launches_note"] = "per rank, counted by the library; NCCL's broadcast kernels not included"
    if rank == 0 and not args.no_cpu_baseline and world == 1:
        result["cpu_baseline"] = cpu_baseline(name, cfg, rp, ci, Xh, elh, erh, args.cpu_seconds)
    g.close()
    torch.cuda.synchronize()
    for p_ in sym_ptrs:
        tlp.tlp_comm_free_symmetric(comm, p_)
    if comm is not None:
        tlp.tlp_comm_destroy(comm)
    if use_dist:
        dist.destroy_process_group()
    if rank == 0:
        print(json.dumps(result))


# ------------------------------------------------------- oracle baselines ---

def _oracle_rows(name, cfg, rp, ci, Xh, elh, erh, rows):
    import oracle
    import synth
    F = cfg["F"]
    by = 0
    t0 = time.perf_counter()
    for op in WORKLOADS[name]["ops"]:
        if op in ("gcn", "gcn_bwd"):  # (bwd: the reddit graph is symmetric, same work per row)
            oracle.gcn(rp, ci, Xh, "both", rows=rows, F=F)
        elif op == "gcn2":
            # layer 2 of a row needs layer 1 at its in-neighbours: the bounded sample
            # times layer 1 on the sampled rows twice (same work per row as layer 2)
            oracle.gcn(rp, ci, Xh, "both", rows=rows, F=F)
            oracle.gcn(rp, ci, Xh, "both", rows=rows, F=F)
        elif op == "gin":
            oracle.gin(rp, ci, Xh, synth.EPS, rows=rows, F=F)
        elif op == "sage":
            oracle.sage(rp, ci, Xh, include_self=True, rows=rows, F=F)
        elif op == "gat":
            oracle.gat(rp, ci, Xh, elh, erh, synth.SLOPE, rows=rows, F=F)
        elif op == "gat_bwd":
            # the backward of the sampled destination rows: the sub-CSR of their
            # in-edges (every gradient term belongs to exactly one such row)
            sub_rp = np.concatenate([[0], np.cumsum(rp[rows + 1] - rp[rows])]).astype(np.int64)
            sub_ci = np.concatenate([ci[rp[v]:rp[v + 1]] for v in rows]).astype(np.int32)
            oracle.gat_backward(sub_rp, sub_ci, Xh, elh, erh[rows], synth.SLOPE, Xh[rows], F=F)
        else:
            H = int(op[3:])
            oracle.gat_mh(rp, ci, Xh, elh, erh, H, synth.SLOPE, rows=rows, Fh=F // H)
        e = int((rp[rows + 1] - rp[rows]).sum())
        by += gather_bytes(op, len(rows), e, F)
    return by, time.perf_counter() - t0


def _calibrated_rows(name, cfg, rp, ci, Xh, elh, erh, seconds, seed=0):
    rng = np.random.default_rng(seed)
    perm = rng.permutation(cfg_n(cfg))
    probe = np.sort(perm[:64])
    by, dt = _oracle_rows(name, cfg, rp, ci, Xh, elh, erh, probe)
    k = int(max(64, min(cfg_n(cfg), 64 * seconds / max(dt, 1e-3))))
    return np.sort(perm[:k])


def _pool_worker(job):
    """One process of the all-core oracle run: its chunk of rows, inputs
    memory-mapped from the shared directory (no copies)."""
    d, name, F, rows = job
    rp = np.load(os.path.join(d, "rp.npy"), mmap_mode="r")
    ci = np.load(os.path.join(d, "ci.npy"), mmap_mode="r")
    Xh = np.load(os.path.join(d, "X.npy"), mmap_mode="r")
    elh = np.load(os.path.join(d, "el.npy"), mmap_mode="r")
    erh = np.load(os.path.join(d, "er.npy"), mmap_mode="r")
    cfg = {"F": F}
    t0 = time.perf_counter()
    by, _ = _oracle_rows(name, cfg, np.asarray(rp), ci, Xh, elh, erh, rows)
    return by, time.perf_counter() - t0


def oracle_all_cores(name, cfg, rp, ci, Xh, elh, erh, rows, cores):
    """The oracle as it stands, on `cores` processes over disjoint row chunks
    (rows are independent, so every output is the single-threaded one, bit for
    bit).  Returns (bytes, wall seconds)."""
    import multiprocessing as mp
    import shutil
    import tempfile
    base = "/dev/shm" if os.path.isdir("/dev/shm") else None
    d = tempfile.mkdtemp(prefix="tlp_oracle_", dir=base)
    try:
        for nm, arr in (("rp", rp), ("ci", ci), ("X", Xh), ("el", elh), ("er", erh)):
            np.save(os.path.join(d, nm + ".npy"), np.ascontiguousarray(arr))
        chunks = [c for c in np.array_split(rows, cores) if len(c)]
        ctx = mp.get_context("spawn")
        with ctx.Pool(len(chunks)) as pool:
            pool.map(_pool_worker, [(d, name, cfg["F"], chunks[0][:2])] * len(chunks))  # warm (imports)
            t0 = time.perf_counter()
            res = pool.map(_pool_worker, [(d, name, cfg["F"], c) for c in chunks])
            wall = time.perf_counter() - t0
        return sum(r[0] for r in res), wall
    finally:
        shutil.rmtree(d, ignore_errors=True)


def cpu_baseline(name, cfg, rp, ci, Xh, elh, erh, seconds):
    """The fp64 oracle, untuned, on the host: single-threaded on a calibrated
    row sample, then on all cores (one process per core, disjoint row chunks)
    on a sample `cores` times larger."""
    cores = len(os.sched_getaffinity(0))
    rows = _calibrated_rows(name, cfg, rp, ci, Xh, elh, erh, seconds / 3)
    by1, dt1 = _oracle_rows(name, cfg, rp, ci, Xh, elh, erh, rows)
    out = {"kind": "oracle", "unit": "GB/s", "cpu_model": cpu_model(),
           "host_cores_available": cores,
           "single_thread": {"value": round(by1 / dt1 / 1e9, 4), "cores": 1,
                             "sample": f"{len(rows)} of {cfg_n(cfg)} destination rows, {dt1:.1f} s"}}
    try:
        rng = np.random.default_rng(1)
        k = int(min(cfg_n(cfg), len(rows) * cores * 0.5))
        big = np.sort(rng.permutation(cfg_n(cfg))[:k])
        byn, dtn = oracle_all_cores(name, cfg, rp, ci, Xh, elh, erh, big, cores)
        out.update({"value": round(byn / dtn / 1e9, 4), "cores": cores,
                    "sample": f"{len(big)} of {cfg_n(cfg)} destination rows (uniform random, seed 1), "
                              f"all ops of the step, {dtn:.1f} s wall on {cores} processes "
                              f"(~{dtn * cores:.0f} s of CPU), fp64 oracle"})
    except Exception as e:  # noqa: BLE001 -- keep the single-thread figure
        out.update({"value": out["single_thread"]["value"], "cores": 1,
                    "sample": out["single_thread"]["sample"], "all_cores_error": repr(e)[:200]})
    return out


def run_reference(args):
    """The oracle as it stands, on the host cores, on this workload's metric."""
    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    if rank != 0:
        return
    name = args.workload
    cfg, rp, ci, Xh, elh, erh = make_inputs(name, "cpu")
    E = len(ci)
    per_step = max(1.0, min(8.0, 150.0 / max(1, args.steps + args.warmup)))
    rows = _calibrated_rows(name, cfg, rp, ci, Xh, elh, erh, per_step)
    for _ in range(args.warmup):
        _oracle_rows(name, cfg, rp, ci, Xh, elh, erh, rows)
    tot_b, tot_t = 0, 0.0
    for _ in range(args.steps):
        b, t = _oracle_rows(name, cfg, rp, ci, Xh, elh, erh, rows)
        tot_b += b
        tot_t += t
    value = tot_b / tot_t / 1e9
    sample = (f"{len(rows)} of {cfg_n(cfg)} destination rows per step (uniform random, seed 0), "
              f"all ops of the step, single-threaded fp64 oracle")
    out = {"impl": "reference", "metric": METRIC, "value": round(value, 4), "unit": "GB/s",
           "n_gpus": world, "steps": args.steps, "warmup": args.warmup,
           "ms_per_step": round(tot_t / args.steps * 1e3, 1), "higher_is_better": True,
           "scaling": "strong", "vs_baseline": None, "dtype": "f64", "data": "synthetic",
           "config": {"workload": workload_desc(name, cfg, E), "parallelism": "host, 1 thread"},
           "cpu_baseline": {"value": round(value, 4), "unit": "GB/s", "cores": 1,
                            "kind": "oracle", "sample": sample},
           "e2e": {"value": round(value, 4), "unit": "GB/s", "h2d_bytes_per_step": 0,
                   "d2h_bytes_per_step": 0},
           "gpu_launches": 0}
    print(json.dumps(out))


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=10)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--impl", default="tlp", choices=["tlp", "reference"])
    ap.add_argument("--workload", default="reddit", choices=sorted(WORKLOADS))
    ap.add_argument("--no-e2e", action="store_true")
    ap.add_argument("--cold", action="store_true",
                    help="also time each op with L2 flushed before it (SURVEY 8(d) d3 cold regime)")
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--cpu-seconds", type=float, default=15.0)
    ap.add_argument("--cuda-graph", action="store_true",
                    help="replay each op as a captured CUDA graph (launch-bound small graphs)")
    ap.add_argument("--graph-reps", type=int, default=20,
                    help="graph replays per timed op with --cuda-graph (times are per replay)")
    ap.add_argument("--fused", action="store_true",
                    help="with --dist/torchrun: NEXT-2 fused compute + all-gather over NVLink peer memory")
    ap.add_argument("--dist", action="store_true",
                    help="use the NCCL dist API even at world size 1 (exercises the N>1 path)")
    ap.add_argument("--spawn", action="store_true",
                    help="start the ranks through torch.distributed.run even for --gpus 1")
    ap.add_argument("--selftest", action="store_true",
                    help="CPU check of the multi-rank launcher (gloo, no GPU): ranks partition "
                         "the Reddit-shaped rows with libtlp's host partition and reduce a time")
    args = ap.parse_args()
    if args.warmup < 3:
        print("warning: the contract wants >= 3 warm-up steps", file=sys.stderr)
    world_env = os.environ.get("WORLD_SIZE")
    if world_env is None and (args.gpus > 1 or args.spawn):
        # --gpus N without a launcher: start N ranks ourselves (one process per
        # GPU, torchrun over 127.0.0.1), forwarding the same arguments
        if not args.selftest and args.impl == "tlp":
            try:
                import torch
                have = torch.cuda.device_count()
            except Exception:
                have = 0
            if have < args.gpus:
                print(f"error: --gpus {args.gpus} but only {have} CUDA device(s) visible", file=sys.stderr)
                sys.exit(1)
        sys.exit(launch_ranks(args.gpus, [a for a in sys.argv[1:] if a != "--spawn"]))
    if world_env is not None and int(world_env) != args.gpus:
        print(f"error: --gpus {args.gpus} but WORLD_SIZE={world_env}", file=sys.stderr)
        sys.exit(2)
    if args.selftest:
        run_selftest(args)
    elif args.impl == "reference":
        run_reference(args)
    else:
        run_tlp(args)


def launch_ranks(n, argv):
    """Re-run this script under torch.distributed.run with n ranks on this node."""
    import socket
    with socket.socket() as sk:
        sk.bind(("127.0.0.1", 0))
        port = sk.getsockname()[1]
    cmd = [sys.executable, "-m", "torch.distributed.run", "--nnodes=1", f"--nproc-per-node={n}",
           "--master-addr=127.0.0.1", f"--master-port={port}", os.path.abspath(__file__)] + list(argv)
    return subprocess.call(cmd)


def run_selftest(args):
    """Launcher self-test on CPU (gloo): every rank computes the edge-balanced
    row bounds with libtlp's host partition (tlp_partition_rows), checks them
    against the oracle's rule, and the max-over-ranks reduction of a time runs
    as in run_tlp; rank 0 prints one JSON line."""
    import torch
    import torch.distributed as dist
    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    import oracle
    import paper_conf_hpdc_fujh22_b200 as tlp
    import synth
    rp, _ = synth.chung_lu(3000, 60000, 0.4, 9, device="cpu")
    b = tlp.tlp_partition_rows(rp, world)
    ok = bool(np.array_equal(b, oracle.partition(rp, world)))
    my_edges = int(rp[b[rank + 1]] - rp[b[rank]])
    t = torch.tensor([float(my_edges)])
    dist.all_reduce(t, op=dist.ReduceOp.MAX)
    tot = torch.tensor([float(my_edges)])
    dist.all_reduce(tot, op=dist.ReduceOp.SUM)
    okt = torch.tensor([1 if ok else 0])
    dist.all_reduce(okt, op=dist.ReduceOp.MIN)
    if rank == 0:
        print(json.dumps({"selftest": "launcher", "n_gpus": world, "bounds_match_oracle": bool(okt.item()),
                          "edges_total": int(tot.item()), "edges_max_rank": int(t.item()),
                          "nnz": int(rp[-1])}))
    dist.destroy_process_group()


if __name__ == "__main__":
    main()

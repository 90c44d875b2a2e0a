/*
 * tlp.h -- C ABI of the B200-native TLPGNN neighbor-aggregation library.
 *
 * The operation (PAPER.md = /root/reference/PAPER.md, "P:<line>"):
 *   Eq. 1-2: a_u = (+)_{v in N(u)} psi(h_u, e_vu, h_v), h'_u = sigma(a_u).
 *   This library computes the graph-convolution phase only ("each
 *   vertex gathers the features of all its neighbors ... combines the results
 *   with its own features, and uses a reduce operation"); sigma and the dense
 *   X*W phase are the caller's (out of scope).
 *   The graph is a destination-major in-edge CSR (Fig. 7, P:1020-1028:
 *   "int start = indptr[des_v]; ... features[indices[i]*F + f]"): the in-edges
 *   of destination row v are e in [rowptr[v], rowptr[v+1]) with source
 *   u = colidx[e].  The structure is static across layers, hence a
 *   create-once handle.
 *
 * Conventions (all calls):
 *   - Return codes only (tlp_status); no exception or abort crosses the ABI.
 *     tlp_last_error() gives a thread-local detail string for the last failure.
 *   - "device pointer" = CUDA device memory of the current device; where a
 *     call says "device or host", any pointer CUDA's unified addressing can copy
 *     from (cudaMemcpyDefault) is accepted.
 *   - `stream` is a cudaStream_t passed as void* (NULL = legacy default
 *     stream).  Aggregations are stream-ordered and never synchronise the host;
 *     a kernel fault surfaces as TLP_ERR_CUDA on a later call.
 *   - Features are row-major fp32 with an explicit leading dimension (row
 *     stride in floats) ld >= F.  Only columns [0, F) of Y are written; pad
 *     columns [F, ld) of Y are never touched (single-GPU calls).
 *   - Ownership: a tlp_graph owns private copies of everything it was created
 *     from; X, Y, el, er are borrowed until the enqueued work completes.
 *   - One in-flight aggregation per handle (its scheduling counters and hub
 *     scratch are shared); handles are not thread-safe.
 *   - Results are bitwise reproducible: every destination row is reduced in a
 *     fixed order (CSR order; hub chunks merged in index order) independent of
 *     scheduling, launch geometry and the number of GPUs.
 */
#ifndef TLP_H
#define TLP_H

#include <stddef.h>
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

#define TLP_VERSION_MAJOR 0
#define TLP_VERSION_MINOR 1

typedef enum tlp_status {
    TLP_OK = 0,
    TLP_ERR_INVALID_ARGUMENT = 1, /* null/negative/size mismatch/overlap/alignment */
    TLP_ERR_INVALID_GRAPH = 2,    /* CSR violates the create contract            */
    TLP_ERR_OUT_OF_MEMORY = 3,
    TLP_ERR_CUDA = 4,             /* a CUDA runtime error (maybe from earlier work) */
    TLP_ERR_NCCL = 5,
    TLP_ERR_UNSUPPORTED = 6
} tlp_status;

/* GCN normalisation ("The sum operation is weighted based on degree",
 * P:1110-1111 "weighted sum"; the formula is not printed, reading R1):
 *   NONE : Y[v] = sum_e w_e X[u]                                (Fig. 7 plain sum)
 *   RIGHT: Y[v] = 1/max(d_in(v),1) * sum_e w_e X[u]             (mean)
 *   BOTH : Y[v] = 1/sqrt(max(d_in(v),1)) * sum_e w_e X[u]/sqrt(max(d_out(u),1))
 *          (Kipf & Welling [26]).  Degrees are unweighted edge counts. */
typedef enum tlp_norm {
    TLP_NORM_NONE = 0,
    TLP_NORM_RIGHT = 1,
    TLP_NORM_BOTH = 2
} tlp_norm;

/* Work scheduling (Section 5 "Hybrid workload balancing").  All modes
 * produce bitwise-identical results; they differ only in speed.
 *   DYNAMIC : persistent grid, static first wave, then atomic-counter fetch of
 *             `step` tasks at a time (Alg. 1)           [default]
 *   STATIC  : persistent grid, task t handled by warp t mod W (no atomics)
 *   HARDWARE: one warp per task, grid sized to the task count
 *   PAPER   : the paper's heuristic switch: DYNAMIC if
 *             n_dst > 1,000,000 or nnz/n_dst > 50, else HARDWARE.
 *   CLC     : Blackwell Cluster Launch Control work stealing:
 *             one CTA per warps_per_cta x step tasks; a running CTA cancels a
 *             not-yet-started CTA (clusterlaunchcontrol.try_cancel) and takes
 *             over its tasks -- Alg. 1's balancing without a global counter. */
typedef enum tlp_sched {
    TLP_SCHED_DYNAMIC = 0,
    TLP_SCHED_STATIC = 1,
    TLP_SCHED_HARDWARE = 2,
    TLP_SCHED_PAPER = 3,
    TLP_SCHED_CLC = 4
} tlp_sched;

/* Aggregation kinds of the descriptor API (tlp_aggregate). */
typedef enum tlp_op {
    TLP_OP_GCN = 0,
    TLP_OP_GIN = 1,
    TLP_OP_GAT = 2,
    TLP_OP_SAGE = 3,   /* GraphSage mean (NEXT-1)      */
    TLP_OP_GAT_MH = 4  /* multi-head GAT (NEXT-1)      */
} tlp_op;

/* Layer activation of the fused epilogue (Eq. 2's sigma; NEXT-3). */
typedef enum tlp_act {
    TLP_ACT_NONE = 0,
    TLP_ACT_RELU = 1,       /* max(x, 0)                         */
    TLP_ACT_LEAKY_RELU = 2, /* x >= 0 ? x : act_param * x        */
    TLP_ACT_ELU = 3         /* x > 0 ? x : act_param * (e^x - 1) */
} tlp_act;

/* One aggregation, fully described (tlp_aggregate / tlp_dist_aggregate).  The
 * fields an op does not use are ignored.  After the reduction the epilogue
 * Y = act(Y + bias) is applied per element in the same kernel (NEXT-3: the
 * "activation" phase of the layer, fused into the store). */
typedef struct tlp_agg_desc {
    int op;                   /* tlp_op                                        */
    const float *X;           /* device [n_src x ldx]                          */
    int64_t F, ldx;
    float *Y;                 /* device [n_dst x ldy] (dist: the full Y)       */
    int64_t ldy;
    int norm;                 /* GCN: tlp_norm                                 */
    float eps;                /* GIN                                           */
    const float *el, *er;     /* GAT: [n_src], [row_offset+n_dst]; GAT_MH: x heads */
    float slope;              /* GAT LeakyReLU slope                           */
    int64_t heads;            /* GAT_MH (0 or 1 = one head)                    */
    int include_self;         /* SAGE                                          */
    const float *bias;        /* epilogue: fp32 device [F] or NULL             */
    int act;                  /* epilogue: tlp_act                             */
    float act_param;          /* LeakyReLU slope / ELU alpha                   */
    /* epilogue projections (NEXT-3, single head, single GPU): after bias and
     * activation, el_out[v] = sum_f Y[v,f] att_l[f] and er_out[v] =
     * sum_f Y[v,f] att_r[f] -- the next GAT layer's attention terms, formed
     * while the row is still in registers (per-strip partials reduced in strip
     * order by one extra launch: deterministic).  att_*: fp32 device [F] or
     * NULL; *_out: fp32 device [n_dst] or NULL (set both of a pair). */
    const float *att_l, *att_r;
    float *el_out, *er_out;
} tlp_agg_desc;

typedef struct tlp_graph_s *tlp_graph;
typedef struct tlp_comm_s *tlp_comm;

/* Plan options for tlp_graph_create_ex (0 = library default).  They change
 * only the work decomposition (and therefore fp32 rounding order), never the
 * mathematical result; they never depend on the GPU count. */
typedef struct tlp_create_opts {
    int64_t hub_threshold; /* H: rows with in-degree > H are split (default 1024) */
    int64_t hub_chunk;     /* C: edges per hub chunk (default 512)               */
    int64_t unit_edges;    /* K: target edges per regular work unit (default 64) */
} tlp_create_opts;

typedef struct tlp_graph_info {
    int64_t n_dst;         /* destination rows of this handle                  */
    int64_t n_src;         /* source vertices (rows of X)                       */
    int64_t nnz;           /* edges of this handle                              */
    int64_t row_offset;    /* global id of local row 0 (0 unless a dist slice)  */
    int64_t max_in_degree;
    int64_t n_hubs;        /* rows with in-degree > hub_threshold               */
    int64_t n_hub_chunks;  /* sum over hubs of ceil(deg / hub_chunk)            */
    int64_t n_units;       /* regular (non-hub) work units                      */
    int64_t n_tasks;       /* n_hub_chunks + n_units                            */
    int64_t hub_threshold, hub_chunk, unit_edges;
    int64_t has_edge_weight;
    int64_t device_bytes;  /* bytes of device memory owned by the handle        */
    int64_t scratch_bytes; /* hub-partial scratch currently allocated           */
    double create_ms;      /* host wall time of the create call                 */
    int64_t launches;      /* kernels enqueued by calls on this handle since
                            * create (aggregations, their pre-/post-passes, the
                            * transposed handle's backward launches); graph
                            * construction and NCCL kernels are not counted   */
} tlp_graph_info;

/* ---- status ------------------------------------------------------------- */
const char *tlp_status_string(tlp_status s);
/* Thread-local detail of the last non-OK status returned on this thread. */
const char *tlp_last_error(void);
/* Returns TLP_VERSION_MAJOR*100 + TLP_VERSION_MINOR. */
int tlp_version(void);

/* ---- graph handle ------------------------------------ */

/* Creates a handle for the in-edge CSR with n_dst rows over n_src sources.
 *   rowptr      : int64 [n_dst+1], device or host
 *   colidx      : int32 [nnz],     device or host
 *   edge_weight : fp32  [nnz] or NULL (w_e = 1), device or host
 * Validates the CSR (rowptr[0] = 0, non-decreasing, rowptr[n_dst] = nnz,
 * 0 <= colidx < n_src), copies it into handle-owned buffers, derives degrees,
 * the BOTH-norm coefficients and the work plan (hub split + units), and
 * synchronises `stream` before returning.  The caller may free its arrays on
 * return.  n_src < 2^31.
 * Errors: TLP_ERR_INVALID_ARGUMENT (null out, negative sizes, null arrays with
 * nnz > 0), TLP_ERR_INVALID_GRAPH, TLP_ERR_OUT_OF_MEMORY, TLP_ERR_CUDA.  On error
 * *out = NULL and nothing is leaked. */
tlp_status tlp_graph_create(int64_t n_dst, int64_t n_src, int64_t nnz,
                            const int64_t *rowptr, const int32_t *colidx,
                            const float *edge_weight, void *stream,
                            tlp_graph *out);

/* As tlp_graph_create with explicit plan options (opts may be NULL). */
tlp_status tlp_graph_create_ex(int64_t n_dst, int64_t n_src, int64_t nnz,
                               const int64_t *rowptr, const int32_t *colidx,
                               const float *edge_weight,
                               const tlp_create_opts *opts, void *stream,
                               tlp_graph *out);

/* Waits for the handle's pending work and frees it.  NULL is a no-op. */
tlp_status tlp_graph_destroy(tlp_graph g);

/* Host-side copy of the handle's sizes and plan statistics. */
tlp_status tlp_graph_info_get(tlp_graph g, tlp_graph_info *out);

/* Copies the derived integer degrees (bit-exact structure tests):
 * in_deg int32 [n_dst], out_deg int32 [n_src] (global over the full CSR for a
 * dist slice).  Either may be NULL.  Device or host destinations; synchronous. */
tlp_status tlp_graph_degrees(tlp_graph g, int32_t *in_deg, int32_t *out_deg,
                             void *stream);

/* Copies the work plan (synchronous; device or host destinations; any may be NULL):
 *   tasks       int32 [2*n_tasks]: pairs (a,b); b >= 0: regular unit of rows
 *               [a,b); b < 0: chunk j = -b-1 of hub index a.  Hub chunks
 *               come first, largest hub first.
 *   hub_rows    int32 [n_hubs]   : local row of each hub, by descending degree
 *   hub_chunk_off int32 [n_hubs+1]: prefix sum of chunks per hub. */
tlp_status tlp_graph_plan(tlp_graph g, int32_t *tasks, int32_t *hub_rows,
                          int32_t *hub_chunk_off, void *stream);

/* Debug visit counter (Alg. 1's exactly-once semantics,
 * P:883-906): while `counter` (device int32 [n_dst], zeroed by the caller) is
 * set, every aggregation on this handle adds 1 to counter[r] each time it
 * finishes one feature strip of local row r -- after a call every row holds
 * exactly the number of strips that call used (hub rows included: their
 * chunk partials are merged, and the row stored, once per strip).  Borrowed
 * until reset with NULL.  Costs one atomic per row strip; off by default. */
tlp_status tlp_graph_set_visit_counter(tlp_graph g, int32_t *counter);

/* Selects the scheduler (tlp_sched), warps per CTA (0 = default 8) and the
 * tasks fetched per atomic (Alg. 1's `step`; 0 = derived from F; CLC: tasks
 * per warp of one CTA's block).  Unknown sched -> TLP_ERR_INVALID_ARGUMENT. */
tlp_status tlp_graph_set_schedule(tlp_graph g, int sched, int warps_per_cta,
                                  int step);

/* ---- aggregations (one kernel launch per call) --------- */

/* GCN: Y[v, 0:F) = c_in(v) * sum_{e in row v} w_e * c_out(colidx[e]) * X[colidx[e], 0:F)
 *   X : fp32 device [n_src x ldx], Y : fp32 device [n_dst x ldy], ld >= F >= 0.
 * F = 0 or n_dst = 0 is a no-op.  X and Y must not overlap. */
tlp_status tlp_gcn_aggregate(tlp_graph g, const float *X, int64_t F,
                             int64_t ldx, int norm, float *Y, int64_t ldy,
                             void *stream);

/* GIN (Xu et al. [51]):
 *   Y[v, 0:F) = (1+eps) * X[row_offset+v, 0:F) + sum_e w_e * X[colidx[e], 0:F)
 * Requires row_offset + n_dst <= n_src. */
tlp_status tlp_gin_aggregate(tlp_graph g, const float *X, int64_t F,
                             int64_t ldx, float eps, float *Y, int64_t ldy,
                             void *stream);

/* GAT, single head ("calculates an attention coefficient for each
 * edge and then aggregates all neighbors' features weighted by the softmax over
 * all attentions"; Velickovic [43]).  For row v with in-degree d:
 *   s_e = LeakyReLU(el[u] + er[row_offset+v], slope)   (x >= 0 ? x : slope*x)
 *   Y[v] = sum_e softmax_e(s) * X[u]      (d = 0: Y[v] = 0)
 * computed in one pass with an online (running max) softmax; scores never
 * leave registers.  el: fp32 device [n_src]; er: fp32 device
 * [row_offset+n_dst].  Edge weights are ignored.
 * When X exceeds L2 but its 64-column strips fit the call
 * instead runs an edge-softmax pre-pass (the oracle's two-pass softmax, alpha_e
 * in a handle-owned buffer) and the streamed-weight sum; the pre-pass runs on
 * a side stream owned by the handle, forked from and joined back into
 * `stream` with events, so the call stays ordered on `stream`. */
tlp_status tlp_gat_aggregate(tlp_graph g, const float *X, int64_t F,
                             int64_t ldx, const float *el, const float *er,
                             float slope, float *Y, int64_t ldy, void *stream);

/* Any aggregation from a descriptor, with the fused layer epilogue
 * act(Y + bias).  Same errors as the specific calls, plus
 * TLP_ERR_INVALID_ARGUMENT for an unknown op or activation. */
tlp_status tlp_aggregate(tlp_graph g, const tlp_agg_desc *desc, void *stream);

/* ---- NEXT-1: GraphSage mean, multi-head GAT ------------------ */

/* GraphSage mean aggregator (Hamilton et al. [15]):
 *   include_self = 0: Y[v] = (1/max(d,1)) * sum_e X[u]            (mean over N(v))
 *   include_self = 1: Y[v] = (X[row_offset+v] + sum_e X[u]) / (d+1) (mean over N(v)+v)
 * Unweighted (edge weights ignored).  The concatenation / linear layer of
 * GraphSage is dense and out of scope.  Same layouts and errors as GCN;
 * include_self requires row_offset + n_dst <= n_src. */
tlp_status tlp_sage_aggregate(tlp_graph g, const float *X, int64_t F,
                              int64_t ldx, int include_self, float *Y,
                              int64_t ldy, void *stream);

/* Multi-head GAT (Velickovic [43]): `heads` independent attention heads; head
 * h owns feature columns [h*F/heads, (h+1)*F/heads) of X and Y (F must be a
 * multiple of heads) and has its own scores and softmax:
 *   s_e,h = LeakyReLU(el[u*heads + h] + er[(row_offset+v)*heads + h], slope)
 * el: fp32 device [n_src x heads], er: fp32 device [(row_offset+n_dst) x heads]
 * (row-major).  heads = 1 equals tlp_gat_aggregate. */
tlp_status tlp_gat_mh_aggregate(tlp_graph g, const float *X, int64_t heads,
                                int64_t F, int64_t ldx, const float *el,
                                const float *er, float slope, float *Y,
                                int64_t ldy, void *stream);

/* ---- NEXT-4: backward aggregation ---------------------------- */

/* Builds (once) the transposed out-edge CSR the backward calls run on (stable
 * sort of the edges by source; each source's edges stay in destination order)
 * with its own degrees and plan.  O(nnz) extra device memory; synchronises
 * `stream`.  Not available for dist row slices (TLP_ERR_UNSUPPORTED). */
tlp_status tlp_graph_build_transpose(tlp_graph g, void *stream);

/* GCN backward (Eq. 1 training): dX = M^T dY for the forward GCN
 * operator M of the same norm, i.e.
 *   dX[u] = sum_{edges e: u -> v} c_in(v) w_e c_out(u) dY[v].
 * dY: fp32 device [n_dst x lddy], dX: fp32 device [n_src x lddx].  Needs
 * tlp_graph_build_transpose.  One kernel launch; deterministic. */
tlp_status tlp_gcn_backward(tlp_graph g, const float *dY, int64_t F,
                            int64_t lddy, int norm, float *dX, int64_t lddx,
                            void *stream);

/* GIN backward: dX[u] = (1+eps) dY[u] + sum_{edges e: u -> v} w_e dY[v]
 * (square graphs). */
tlp_status tlp_gin_backward(tlp_graph g, const float *dY, int64_t F,
                            int64_t lddy, float eps, float *dX, int64_t lddx,
                            void *stream);

/* GAT backward (single head; the training workload of the attention layer,
 * P:1001-1007 / Velickovic [43]).  Forward: t_e = el[u] + er[v],
 * s_e = LeakyReLU(t_e, slope), alpha_e = softmax of s_e over the in-edges of v,
 * Y[v] = sum_e alpha_e X[u].  Given dY = dL/dY it writes
 *   dX[u]  = sum_{edges e: u -> v} alpha_e dY[v]                 [n_src x lddx]
 *   del[u] = sum_{edges e: u -> v} dt_e,  der[v] = sum_{e in v} dt_e,
 *   dt_e   = alpha_e (dY[v].X[u] - dY[v].Y[v]) (t_e >= 0 ? 1 : slope).
 * X: fp32 device [n_src x ldx]; el [n_src], er [n_dst], del [n_src], der [n_dst]
 * fp32 device; Y: the forward output of tlp_gat_aggregate for the same inputs,
 * [n_dst x ldy]; dY [n_dst x lddy].  Needs tlp_graph_build_transpose.  Five
 * launches (softmax state per destination, edge weights alpha_e in transposed
 * order, the fused dX + edge-dot aggregation on the transposed CSR, two
 * per-row reductions), stream-ordered, deterministic.  Scratch:
 * n_dst*16 + 2*nnz*4 bytes on the handle and (strips x nnz x 4) bytes on its
 * transpose, grown on demand.  F = 0 writes del = der = 0. */
tlp_status tlp_gat_backward(tlp_graph g, const float *X, int64_t F, int64_t ldx,
                            const float *el, const float *er, float slope,
                            const float *Y, int64_t ldy, const float *dY,
                            int64_t lddy, float *dX, int64_t lddx, float *del,
                            float *der, void *stream);

/* ---- multi-GPU (destination-row ranges balanced by edge count) ------------ */

/* Pure host function: bounds[0] = 0, bounds[parts] = n, and for 0 < k < parts
 * bounds[k] = min{ r in [0,n] : rowptr[r] >= floor(k*nnz/parts) },
 * nnz = rowptr[n].  rowptr_host: int64 [n+1] host; bounds_host: int64 [parts+1]. */
tlp_status tlp_partition_rows(const int64_t *rowptr_host, int64_t n, int parts,
                              int64_t *bounds_host);

/* Handle for the destination rows [row_begin, row_end) of a full square CSR
 * (n x n; rowptr int64 [n+1], colidx int32 [nnz], device or host): local row i
 * is global row row_begin + i (info.row_offset = row_begin), sources stay
 * global, out-degrees are counted over the whole CSR.  The building block of
 * the dist layer; also lets a single process emulate any partition. */
tlp_status tlp_graph_create_rows(int64_t n, int64_t nnz, const int64_t *rowptr,
                                 const int32_t *colidx, const float *edge_weight,
                                 int64_t row_begin, int64_t row_end,
                                 const tlp_create_opts *opts, void *stream,
                                 tlp_graph *out);

/* NCCL communicator owned by the library (NCCL 2.28, one process per GPU).
 * The unique id (128 bytes) is produced on one rank and broadcast by the
 * caller (e.g. through torch.distributed). */
tlp_status tlp_comm_get_unique_id(uint8_t id[128]);
tlp_status tlp_comm_create(const uint8_t id[128], int world, int rank,
                           tlp_comm *out);
tlp_status tlp_comm_destroy(tlp_comm c);

/* Failure detection (the paper is single-GPU, so this
 * follows NCCL's own error model).  tlp_comm_async_error polls the
 * communicator's asynchronous error state without blocking: *nccl_result =
 * the ncclResult_t (0 = ncclSuccess, 7 = ncclInProgress); returns
 * TLP_ERR_NCCL when it is an error.  tlp_comm_abort tears the communicator
 * down without waiting for peers (ncclCommAbort); afterwards only
 * tlp_comm_destroy may be called on it, and dist calls return TLP_ERR_NCCL.
 * tlp_comm_wait blocks until `stream` has drained, polling the error state
 * every ~0.2 ms; on an error, or after timeout_s seconds (<= 0: no limit), it
 * aborts the communicator and returns TLP_ERR_NCCL -- a dead or hung peer
 * cannot hang this rank forever. */
tlp_status tlp_comm_async_error(tlp_comm c, int *nccl_result);
tlp_status tlp_comm_abort(tlp_comm c);
tlp_status tlp_comm_wait(tlp_comm c, void *stream, double timeout_s);

/* Every rank passes the FULL square CSR (n x n, device or host).  The handle
 * holds this rank's row slice [b_k, b_{k+1}) (row_offset = b_k) with
 * out-degrees taken over the full CSR. */
tlp_status tlp_dist_graph_create(tlp_comm c, int64_t n, int64_t nnz,
                                 const int64_t *rowptr, const int32_t *colidx,
                                 const float *edge_weight,
                                 const tlp_create_opts *opts, void *stream,
                                 tlp_graph *out_local);

/* NEXT-2: symmetric output buffers.  Collective over the communicator: every
 * rank allocates `bytes` of device memory visible to every other rank of the
 * node over NVLink.  Preferred form: NCCL's symmetric window (ncclMemAlloc +
 * ncclCommWindowRegister(NCCL_WIN_COLL_SYMMETRIC) + ncclDevCommCreate), whose
 * LSA pointers address every peer's copy and, where the node supports NVLS,
 * whose multicast address lets one multimem store reach all of them; if any
 * of that is unavailable (or TLP_SYM=ipc), a cudaMalloc'd buffer mapped into
 * every peer through CUDA IPC.  *local = this rank's buffer. */
tlp_status tlp_comm_alloc_symmetric(tlp_comm c, size_t bytes, void **local);
/* Collective: unmaps, barriers, frees. */
tlp_status tlp_comm_free_symmetric(tlp_comm c, void *local);
/* Which form a symmetric buffer took: *kind = 0 CUDA IPC, 1 NCCL window (LSA
 * peer pointers), 2 NCCL window with an NVLS multicast address. */
tlp_status tlp_comm_symmetric_kind(tlp_comm c, void *local, int *kind);

/* Copies the partition bounds (int64 [world+1], host). */
tlp_status tlp_dist_bounds(tlp_graph local, int64_t *bounds_host);

/* All-gather of row slabs: rank r's rows [b_r, b_{r+1}) of Y_full (n x ldy,
 * device) are broadcast in place to every rank (grouped ncclBroadcast; NCCL
 * has no all-gatherv).  Whole rows including pad columns are transferred. */
tlp_status tlp_dist_allgather_rows(tlp_graph local, tlp_comm c, float *Y_full,
                                   int64_t ldy, void *stream);

/* Local aggregation of this rank's rows into Y_full + b_k*ldy followed by
 * tlp_dist_allgather_rows.  X_full (and el) are replicated [n x ldx]; er is
 * the full [n] vector.  On stream completion Y_full is identical on every rank
 * and bitwise equal to the single-GPU result. */
tlp_status tlp_dist_gcn_aggregate(tlp_graph local, tlp_comm c,
                                  const float *X_full, int64_t F, int64_t ldx,
                                  int norm, float *Y_full, int64_t ldy,
                                  void *stream);
tlp_status tlp_dist_gin_aggregate(tlp_graph local, tlp_comm c,
                                  const float *X_full, int64_t F, int64_t ldx,
                                  float eps, float *Y_full, int64_t ldy,
                                  void *stream);
tlp_status tlp_dist_gat_aggregate(tlp_graph local, tlp_comm c,
                                  const float *X_full, int64_t F, int64_t ldx,
                                  const float *el, const float *er, float slope,
                                  float *Y_full, int64_t ldy, void *stream);
/* NEXT-2 fused compute + all-gather: desc->Y must be a symmetric buffer
 * (tlp_comm_alloc_symmetric) holding Y_full [n x ldy].  ONE kernel computes this
 * rank's rows and stores each finished row vector into Y_full on every rank
 * over NVLink, overlapping the exchange with the gather.  A one-element NCCL
 * all-reduce on `stream` before the kernel (no rank stores into a peer's
 * Y_full while that peer's earlier work may still read it) and one after it
 * (every rank's stores have landed) order the call.  Same result, bit for
 * bit, as tlp_dist_aggregate. */
tlp_status tlp_dist_aggregate_fused(tlp_graph local, tlp_comm c,
                                    const tlp_agg_desc *desc, void *stream);

/* Test hook of the multi-destination epilogue (single GPU): the aggregation
 * stores every output row into each of the n device buffers listed in
 * dests_host (host array), at the row's global index.  Synchronous. */
tlp_status tlp_debug_multi_store(tlp_graph g, const tlp_agg_desc *desc,
                                 float *const *dests_host, int n, void *stream);

/* Descriptor form of the dist calls (desc->Y is Y_full). */
tlp_status tlp_dist_aggregate(tlp_graph local, tlp_comm c,
                              const tlp_agg_desc *desc, void *stream);
tlp_status tlp_dist_sage_aggregate(tlp_graph local, tlp_comm c,
                                   const float *X_full, int64_t F, int64_t ldx,
                                   int include_self, float *Y_full, int64_t ldy,
                                   void *stream);
tlp_status tlp_dist_gat_mh_aggregate(tlp_graph local, tlp_comm c,
                                     const float *X_full, int64_t heads,
                                     int64_t F, int64_t ldx, const float *el,
                                     const float *er, float slope,
                                     float *Y_full, int64_t ldy, void *stream);

#ifdef __cplusplus
}
#endif
#endif /* TLP_H */

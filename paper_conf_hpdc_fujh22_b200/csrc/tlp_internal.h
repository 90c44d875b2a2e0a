// tlp_internal.h -- private structures of libtlp (not part of the C ABI).
#pragma once

#include <cuda_runtime.h>
#include <stdint.h>

#include <string>

#include "tlp.h"

namespace tlp {

// Defaults of the work plan.  Functions of
// nothing but these constants: never of the GPU count, SM count or timing, so
// the reduction order of every row is partition- and schedule-invariant.
constexpr int64_t kDefaultHubThreshold = 1024;  // H
constexpr int64_t kDefaultHubChunk = 512;       // C
constexpr int64_t kDefaultUnitEdges = 64;       // K
constexpr int kNormLeft = 3;  // internal: per-source 1/max(d_out(u),1), no row scale

// Thread-local error detail; returns `s` for chaining.
tlp_status set_error(tlp_status s, const std::string &msg);
tlp_status cuda_error(cudaError_t e, const char *what);

#define TLP_CUDA_TRY(expr)                                      \
    do {                                                        \
        cudaError_t _e = (expr);                                \
        if (_e != cudaSuccess) return ::tlp::cuda_error(_e, #expr); \
    } while (0)

}  // namespace tlp

// The opaque handle.  All pointers are device memory owned by the handle.
struct tlp_graph_s {
    int64_t n_dst = 0, n_src = 0, nnz = 0, row_offset = 0;
    int device = 0;
    int num_sms = 0;
    int64_t max_in_degree = 0;
    int64_t H = 0, C = 0, K = 0;

    int64_t *rowptr = nullptr;   // [n_dst+1], rowptr[0] = 0
    int32_t *colidx = nullptr;   // [nnz]
    float *ew = nullptr;         // [nnz] or null
    int32_t *in_deg = nullptr;   // [n_dst]
    int32_t *out_deg = nullptr;  // [n_src] (global for a dist slice)
    float *c_out = nullptr;      // [n_src] 1/sqrt(max(out_deg,1))
    float *ew_both = nullptr;    // [nnz] c_out[colidx[e]] * w_e (weighted GCN BOTH coefficient)
    float *xs = nullptr;         // unweighted GCN BOTH: X' = c_out (.) X  [n_src x ldx]
    size_t xs_bytes = 0;
    float *c_out_left = nullptr; // [n_src] 1/max(out_deg,1) (internal LEFT norm, backward of RIGHT)
    tlp_graph_s *t = nullptr;    // transposed graph (tlp_graph_build_transpose), owned
    // source-reuse tags: colidx with the
    // out-degree class of each source in bits 27-31, built on first use
    int32_t *colidx_tag = nullptr;   // [nnz] or null
    int32_t *tpos = nullptr;         // [nnz] forward edge -> transposed position (with t)
    float *bwd = nullptr;            // GAT backward scratch (see tlp_gat_backward)
    size_t bwd_bytes = 0;
    float *proj = nullptr;           // epilogue projection partials [strips x n_dst x 2]
    size_t proj_bytes = 0;
    float *galpha = nullptr;         // GAT edge softmax alpha_e (k_gat_alpha) [nnz]
    size_t galpha_bytes = 0;
    // GAT alpha mode: the edge-softmax pre-pass runs on a forked side stream,
    // concurrently with the gather-copy repack of X (created on first use)
    cudaStream_t side = nullptr;
    cudaEvent_t ev_fork = nullptr, ev_join = nullptr;
    int64_t tag_hist[32] = {0};      // sources per out-degree class

    int2 *tasks = nullptr;       // [n_tasks]
    int32_t *hub_row = nullptr;  // [n_hubs]
    int32_t *hub_off = nullptr;  // [n_hubs+1]
    unsigned int *ctr = nullptr;    // [2]: next task, finished warps
    int64_t n_tasks = 0, n_units = 0, n_hubs = 0, n_chunks = 0;
    int64_t regular_edges = 0;

    float *scratch = nullptr;    // hub partials, GAT (m, den), hub tickets
    size_t scratch_bytes = 0;
    size_t ticket_off = 0, ticket_n = 0;  // ticket region inside scratch (zeroed)
    size_t l2_bytes = 0;
    size_t device_bytes = 0;
    double create_ms = 0.0;
    int64_t launches = 0;        // kernels enqueued by calls on this handle (after create)

    int32_t *visits = nullptr;   // debug visit counter (tlp_graph_set_visit_counter), borrowed
    int sched = TLP_SCHED_DYNAMIC;
    int warps_per_cta = 8;
    int step = 0;

    // dist slice bookkeeping
    int world = 1, rank = 0;
    int64_t *bounds_host = nullptr;  // [world+1] or null
    int64_t n_global = 0;
    cudaStream_t last_stream = nullptr;
};

struct tlp_comm_s;

namespace tlp {

// Internal create used by both the single-GPU and the dist entry points.
//   rowptr/colidx/ew describe rows [row_begin, row_end) of a CSR whose
//   rowptr values are absolute (rebased by rowptr[row_begin]); out-degrees
//   are counted over full_colidx[0:full_nnz) (the full CSR).
tlp_status graph_create_impl(int64_t n_dst, int64_t n_src, int64_t nnz,
                             const int64_t *rowptr, const int32_t *colidx,
                             const float *ew, const int32_t *full_colidx,
                             int64_t full_nnz, int64_t row_offset,
                             const tlp_create_opts *opts, cudaStream_t s,
                             tlp_graph *out);

tlp_status ensure_scratch(tlp_graph g, size_t bytes, cudaStream_t s);
// unweighted graphs: build ew_both[e] = c_out[colidx[e]] on first use (stream-ordered)
tlp_status ensure_edge_both(tlp_graph g, cudaStream_t s);
tlp_status build_transpose(tlp_graph g, cudaStream_t s);

// Enqueue one aggregation kernel; op: 0 GCN, 1 GIN, 2 GAT, 3 GraphSage mean,
// 4 multi-head GAT.
struct AggRequest {
    int op = 0;
    const float *X = nullptr;
    int64_t F = 0, ldx = 0;
    float *Y = nullptr;
    int64_t ldy = 0;
    int norm = 0;
    float eps = 0.f;
    const float *el = nullptr, *er = nullptr;
    float slope = 0.f;
    int sage_self = 0;  // op 3 (GraphSage mean): include the self row
    int64_t heads = 1;  // op 4 (multi-head GAT)
    const float *bias = nullptr;  // layer epilogue: y = act(y + bias)
    int act = 0;
    float act_param = 0.f;
    float *const *dests = nullptr;  // fused all-gather destinations (device array)
    int n_dests = 0;
    float *mc = nullptr;            // NVLS multicast address of Y_full (NCCL window), or null
    // epilogue projections (NEXT-3): el_out = Y.att_l, er_out = Y.att_r
    const float *att_l = nullptr, *att_r = nullptr;
    float *el_out = nullptr, *er_out = nullptr;
    // op 5 (GAT backward on the transposed graph, NEXT-4): X = dY, Y = dX,
    // alpha = edge softmax weights in transposed edge order, xself = forward X;
    // aggregate() allocates the per-strip edge dot products gbuf
    // [n_strips x nnz] and reports them.
    const float *alpha = nullptr;
    const float *xself = nullptr;
    int64_t ldxs = 0;
    float **gbuf_out = nullptr;
    int *n_strips_out = nullptr;
};

inline AggRequest request_from_desc(const tlp_agg_desc &d) {
    AggRequest r;
    r.op = d.op;
    r.X = d.X; r.F = d.F; r.ldx = d.ldx; r.Y = d.Y; r.ldy = d.ldy;
    r.norm = d.norm; r.eps = d.eps;
    r.el = d.el; r.er = d.er; r.slope = d.slope; r.heads = d.heads > 0 ? d.heads : 1;
    r.sage_self = d.include_self;
    r.bias = d.bias; r.act = d.act; r.act_param = d.act_param;
    r.att_l = d.att_l; r.att_r = d.att_r; r.el_out = d.el_out; r.er_out = d.er_out;
    return r;
}
tlp_status aggregate(tlp_graph g, const AggRequest &r, cudaStream_t s);

}  // namespace tlp

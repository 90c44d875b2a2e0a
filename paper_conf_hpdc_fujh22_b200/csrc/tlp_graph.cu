// tlp_graph.cu -- graph handle: ingest + validate, degrees and
// normalisation coefficients (a2), degree-aware work plan (a3).
//
// Create-time work is O(n + nnz) integer passes (the paper's "no
// pre-processing" rule): no reordering, no partition
// building beyond a row-range plan.
#include <cub/cub.cuh>

#include <algorithm>
#include <chrono>
#include <cstdio>
#include <cstring>
#include <string>

#include "tlp_internal.h"

namespace tlp {

static thread_local std::string g_last_error;

tlp_status set_error(tlp_status s, const std::string &msg) {
    g_last_error = msg;
    return s;
}

tlp_status cuda_error(cudaError_t e, const char *what) {
    std::string m = std::string(what) + ": " + cudaGetErrorName(e) + " (" +
                    cudaGetErrorString(e) + ")";
    if (e == cudaErrorMemoryAllocation) return set_error(TLP_ERR_OUT_OF_MEMORY, m);
    return set_error(TLP_ERR_CUDA, m);
}

// ---------------------------------------------------------------- kernels --

enum : int { ERR_ROWPTR0 = 1, ERR_MONO = 2, ERR_LAST = 4, ERR_COL = 8 };

// Copy + rebase the row offsets and check them (a1).
__global__ void k_rowptr_ingest(const int64_t *__restrict__ src, int64_t n_dst,
                                int64_t nnz, int64_t *__restrict__ dst,
                                int32_t *__restrict__ in_deg, int *err) {
    const int64_t base = src[0];
    for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i <= n_dst;
         i += (int64_t)gridDim.x * blockDim.x) {
        int64_t v = src[i] - base;
        dst[i] = v;
        if (i < n_dst) {
            int64_t d = src[i + 1] - src[i];
            if (d < 0) atomicOr(err, ERR_MONO);
            in_deg[i] = (int32_t)d;
        } else if (v != nnz) {
            atomicOr(err, ERR_LAST);
        }
    }
}

// colidx range check and the exact integer out-degree histogram (a2).
__global__ void k_colidx_check(const int32_t *__restrict__ colidx, int64_t nnz,
                               int64_t n_src, int *err) {
    int bad = 0;
    for (int64_t e = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; e < nnz;
         e += (int64_t)gridDim.x * blockDim.x) {
        int32_t u = colidx[e];
        bad |= (u < 0) | ((int64_t)u >= n_src);
    }
    if (__any_sync(0xffffffffu, bad) && (threadIdx.x & 31) == 0) atomicOr(err, ERR_COL);
}

__global__ void k_out_degree(const int32_t *__restrict__ colidx, int64_t nnz,
                             int32_t *__restrict__ out_deg) {
    // 8 independent index loads in flight per thread before their fire-and-
    // forget reductions (the loads cannot be hoisted across the atomics by the
    // compiler on its own)
    constexpr int UN = 8;
    const int64_t stride = (int64_t)gridDim.x * blockDim.x;
    for (int64_t b = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; b < nnz; b += stride * UN) {
        int32_t u[UN];
#pragma unroll
        for (int k = 0; k < UN; ++k) u[k] = (b + k * stride < nnz) ? __ldg(colidx + b + k * stride) : -1;
#pragma unroll
        for (int k = 0; k < UN; ++k)
            if (u[k] >= 0) atomicAdd(&out_deg[u[k]], 1);  // integer: exact in any order
    }
}

// c_out[u] = 1/sqrt(max(out_deg,1)) (BOTH norm, Kipf [26]; R1) and
// c_out_left[u] = 1/max(out_deg,1) (the backward of the RIGHT norm).
__global__ void k_norm(const int32_t *__restrict__ out_deg, int64_t n,
                       float *__restrict__ c_out, float *__restrict__ c_out_left) {
    for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n;
         i += (int64_t)gridDim.x * blockDim.x) {
        int32_t d = out_deg[i];
        const float dc = (float)(d > 1 ? d : 1);
        c_out[i] = 1.0f / sqrtf(dc);
        c_out_left[i] = 1.0f / dc;
    }
}

// Destination row of every edge (transpose build).
__global__ void k_edge_rows(const int64_t *__restrict__ rowptr, int64_t n,
                            int32_t *__restrict__ dst) {
    for (int64_t r = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; r < n;
         r += (int64_t)gridDim.x * blockDim.x)
        for (int64_t e = rowptr[r]; e < rowptr[r + 1]; ++e) dst[e] = (int32_t)r;
}

__global__ void k_iota(int32_t *__restrict__ v, int64_t n) {
    for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n;
         i += (int64_t)gridDim.x * blockDim.x)
        v[i] = (int32_t)i;
}

__global__ void k_permute_edges(const int32_t *__restrict__ perm, int64_t nnz,
                                const int32_t *__restrict__ dst, const float *__restrict__ ew,
                                int32_t *__restrict__ t_col, float *__restrict__ t_ew,
                                int32_t *__restrict__ tpos) {
    for (int64_t k = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; k < nnz;
         k += (int64_t)gridDim.x * blockDim.x) {
        const int32_t e = perm[k];
        t_col[k] = dst[e];
        if (ew) t_ew[k] = ew[e];
        tpos[e] = (int32_t)k;  // inverse permutation (GAT backward)
    }
}

__global__ void k_deg_to_rowptr_input(const int32_t *__restrict__ deg, int64_t n,
                                      int64_t *__restrict__ out) {
    for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i <= n;
         i += (int64_t)gridDim.x * blockDim.x)
        out[i] = (i < n) ? (int64_t)deg[i] : 0;
}

// Per-edge GCN-BOTH coefficient c_out[colidx[e]] * w_e (a2): a coalesced
// stream for the aggregation instead of a dependent gather of c_out.
__global__ void k_edge_both(const int32_t *__restrict__ colidx, const float *__restrict__ ew,
                            const float *__restrict__ c_out, int64_t nnz, float *__restrict__ out) {
    for (int64_t e = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; e < nnz;
         e += (int64_t)gridDim.x * blockDim.x) {
        float c = c_out[colidx[e]];
        if (ew) c *= ew[e];
        out[e] = c;
    }
}

// Plan flags (a3).  Row r starts a work unit iff it is row 0, a hub, follows a
// hub, or a multiple of K edges falls in (rowptr[r-1], rowptr[r]] -- i.e. r is
// lower_bound(rowptr, u*K) for some u.  Hubs (deg > H) become chunk tasks.
__global__ void k_plan_flags(const int64_t *__restrict__ rowptr, int64_t n,
                             int64_t K, int64_t H, uint8_t *__restrict__ start,
                             uint8_t *__restrict__ hub) {
    for (int64_t r = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; r < n;
         r += (int64_t)gridDim.x * blockDim.x) {
        int64_t a = rowptr[r], b = rowptr[r + 1];
        bool is_hub = (b - a) > H;
        // ... or every 256th row, which bounds a unit's row count when long
        // runs of zero-degree rows occur
        bool s = (r == 0) || is_hub || (r % 256 == 0);
        if (r > 0) {
            int64_t p = rowptr[r - 1];
            s = s || ((a - p) > H) || (a / K > p / K);
        }
        start[r] = s;
        hub[r] = is_hub;
    }
}

// Regular tasks from the unit starts; hub units are dropped (flag 0).
__global__ void k_units_to_tasks(const int32_t *__restrict__ starts, int64_t n_units,
                                 int64_t n, const uint8_t *__restrict__ hub,
                                 int2 *__restrict__ out, uint8_t *__restrict__ keep) {
    for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n_units;
         i += (int64_t)gridDim.x * blockDim.x) {
        int32_t r0 = starts[i];
        int32_t r1 = (i + 1 < n_units) ? starts[i + 1] : (int32_t)n;
        out[i] = make_int2(r0, r1);
        keep[i] = !hub[r0];
    }
}

__global__ void k_hub_chunks(const int32_t *__restrict__ hub_deg, int64_t n_hubs,
                             int64_t C, int32_t *__restrict__ nchunk) {
    for (int64_t h = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; h < n_hubs;
         h += (int64_t)gridDim.x * blockDim.x)
        nchunk[h] = (int32_t)((hub_deg[h] + C - 1) / C);
}

__global__ void k_hub_tasks(const int32_t *__restrict__ hub_off, int64_t n_hubs,
                            int2 *__restrict__ tasks) {
    for (int64_t h = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; h < n_hubs;
         h += (int64_t)gridDim.x * blockDim.x)
        for (int32_t j = hub_off[h]; j < hub_off[h + 1]; ++j)
            tasks[j] = make_int2((int32_t)h, -(j - hub_off[h]) - 1);
}

__global__ void k_gather_deg(const int32_t *__restrict__ rows, int64_t n,
                             const int32_t *__restrict__ in_deg, int32_t *__restrict__ out) {
    for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n;
         i += (int64_t)gridDim.x * blockDim.x)
        out[i] = in_deg[rows[i]];
}

// ------------------------------------------------------------- host side --

static int grid_for(int64_t n, int num_sms) {
    int64_t b = (n + 255) / 256;
    int64_t cap = (int64_t)num_sms * 8;
    if (b > cap) b = cap;
    if (b < 1) b = 1;
    return (int)b;
}

namespace {
// Temporary device buffer: stream-ordered allocation from the device's default
// memory pool, freed stream-ordered (no implicit device synchronisation).
struct DevBuf {
    void *p = nullptr;
    cudaStream_t st = nullptr;
    cudaError_t alloc(size_t n, cudaStream_t s) {
        st = s;
        return cudaMallocAsync(&p, n ? n : 16, s);
    }
    ~DevBuf() { if (p) cudaFreeAsync(p, st); }
    template <class T> T *as() { return static_cast<T *>(p); }
};
}  // namespace

static tlp_status dmalloc(void **p, size_t bytes, tlp_graph g) {
    if (bytes == 0) bytes = 16;
    cudaError_t e = cudaMalloc(p, bytes);
    if (e != cudaSuccess) return cuda_error(e, "cudaMalloc");
    if (g) g->device_bytes += bytes;
    return TLP_OK;
}

static void graph_free(tlp_graph g) {
    if (!g) return;
    if (g->t) graph_free(g->t);
    if (g->side) {
        cudaStreamSynchronize(g->side);
        cudaStreamDestroy(g->side);
    }
    if (g->ev_fork) cudaEventDestroy(g->ev_fork);
    if (g->ev_join) cudaEventDestroy(g->ev_join);
    void *ptrs[] = {g->rowptr, g->colidx, g->ew, g->in_deg, g->out_deg, g->c_out, g->ew_both,
                    g->c_out_left, g->colidx_tag, g->tpos, g->bwd, g->proj, g->xs, g->galpha,
                    g->tasks, g->hub_row, g->hub_off, g->ctr,
                    g->scratch};
    for (void *p : ptrs)
        if (p) cudaFree(p);
    delete[] g->bounds_host;
    delete g;
}

#define TRY(expr)                                 \
    do {                                          \
        tlp_status _s = (expr);                   \
        if (_s != TLP_OK) { graph_free(g); return _s; } \
    } while (0)
#define CTRY(expr)                                              \
    do {                                                        \
        cudaError_t _e = (expr);                                \
        if (_e != cudaSuccess) { graph_free(g); return cuda_error(_e, #expr); } \
    } while (0)

tlp_status graph_create_impl(int64_t n_dst, int64_t n_src, int64_t nnz,
                             const int64_t *rowptr, const int32_t *colidx,
                             const float *ew, const int32_t *full_colidx,
                             int64_t full_nnz, int64_t row_offset,
                             const tlp_create_opts *opts, cudaStream_t s,
                             tlp_graph *out) {
    auto t0 = std::chrono::steady_clock::now();
    // TLP_TRACE_CREATE=1: synchronise and print the elapsed time at each phase
    static const bool trace = getenv("TLP_TRACE_CREATE") != nullptr;
    auto mark = [&](const char *what) {
        if (!trace) return;
        cudaStreamSynchronize(s);
        const double ms = std::chrono::duration<double, std::milli>(
                              std::chrono::steady_clock::now() - t0).count();
        fprintf(stderr, "[tlp create] %-28s %9.3f ms\n", what, ms);
    };
    if (!out) return set_error(TLP_ERR_INVALID_ARGUMENT, "out is NULL");
    *out = nullptr;
    if (n_dst < 0 || n_src < 0 || nnz < 0 || row_offset < 0)
        return set_error(TLP_ERR_INVALID_ARGUMENT, "negative size");
    if (n_src >= (int64_t(1) << 31) || n_dst >= (int64_t(1) << 31))
        return set_error(TLP_ERR_INVALID_ARGUMENT, "n_src and n_dst must be < 2^31");
    if (!rowptr) return set_error(TLP_ERR_INVALID_ARGUMENT, "rowptr is NULL");
    if (nnz > 0 && !colidx) return set_error(TLP_ERR_INVALID_ARGUMENT, "colidx is NULL");
    if (nnz > 0 && n_src == 0)
        return set_error(TLP_ERR_INVALID_GRAPH, "edges present but n_src = 0");

    tlp_graph g = new tlp_graph_s();
    CTRY(cudaGetDevice(&g->device));
    CTRY(cudaDeviceGetAttribute(&g->num_sms, cudaDevAttrMultiProcessorCount, g->device));
    {
        int l2 = 0;
        CTRY(cudaDeviceGetAttribute(&l2, cudaDevAttrL2CacheSize, g->device));
        g->l2_bytes = (size_t)l2;
    }
    g->n_dst = n_dst;
    g->n_src = n_src;
    g->nnz = nnz;
    g->row_offset = row_offset;
    g->H = (opts && opts->hub_threshold > 0) ? opts->hub_threshold : kDefaultHubThreshold;
    g->C = (opts && opts->hub_chunk > 0) ? opts->hub_chunk : kDefaultHubChunk;
    if (opts && opts->unit_edges > 0) {
        g->K = opts->unit_edges;
    } else {
        // enough units to give every resident warp (~SMs x 32) about four of
        // them, at most kDefaultUnitEdges edges each.  K only groups whole rows
        // into tasks; it never changes any row's reduction order.
        const int64_t target = (int64_t)std::max(g->num_sms, 1) * 32 * 4;
        g->K = std::max<int64_t>(1, std::min<int64_t>(kDefaultUnitEdges, nnz / target));
    }
    g->last_stream = s;
    const int nsm = g->num_sms;

    mark("setup");
    // ---- a1: ingest (copy; rebased rowptr) and validate -------------------
    TRY(dmalloc((void **)&g->rowptr, sizeof(int64_t) * (n_dst + 1), g));
    TRY(dmalloc((void **)&g->in_deg, sizeof(int32_t) * n_dst, g));
    // colidx with 16 B of slack so vector index loads never leave the buffer
    TRY(dmalloc((void **)&g->colidx, sizeof(int32_t) * nnz + 16, g));
    if (nnz) CTRY(cudaMemcpyAsync(g->colidx, colidx, sizeof(int32_t) * nnz, cudaMemcpyDefault, s));
    if (ew) {
        TRY(dmalloc((void **)&g->ew, sizeof(float) * nnz + 16, g));
        if (nnz) CTRY(cudaMemcpyAsync(g->ew, ew, sizeof(float) * nnz, cudaMemcpyDefault, s));
    }
    DevBuf rp_src, err;
    // rowptr may be host memory: stage it in device memory first
    {
        cudaPointerAttributes attr;
        cudaError_t e = cudaPointerGetAttributes(&attr, rowptr);
        bool on_dev = (e == cudaSuccess) && (attr.type == cudaMemoryTypeDevice ||
                                             attr.type == cudaMemoryTypeManaged);
        if (e != cudaSuccess) cudaGetLastError();
        const int64_t *rp_dev = rowptr;
        if (!on_dev) {
            CTRY(rp_src.alloc(sizeof(int64_t) * (n_dst + 1), s));
            CTRY(cudaMemcpyAsync(rp_src.p, rowptr, sizeof(int64_t) * (n_dst + 1),
                                 cudaMemcpyDefault, s));
            rp_dev = rp_src.as<int64_t>();
        }
        CTRY(err.alloc(sizeof(int), s));
        CTRY(cudaMemsetAsync(err.p, 0, sizeof(int), s));
        // rowptr[0] must be the start of the slice: for a whole graph it must be 0
        int64_t first = 0;
        CTRY(cudaMemcpyAsync(&first, rp_dev, sizeof(int64_t), cudaMemcpyDefault, s));
        k_rowptr_ingest<<<grid_for(n_dst + 1, nsm), 256, 0, s>>>(rp_dev, n_dst, nnz, g->rowptr,
                                                                  g->in_deg, err.as<int>());
        CTRY(cudaGetLastError());
        // a row slice validates the whole CSR it was cut from: its out-degree
        // histogram (a2) indexes out_deg with every source of full_colidx
        const int32_t *chk = full_colidx ? full_colidx : g->colidx;
        const int64_t chk_n = full_colidx ? full_nnz : nnz;
        if (chk_n) {
            k_colidx_check<<<grid_for(chk_n, nsm), 256, 0, s>>>(chk, chk_n, n_src, err.as<int>());
            CTRY(cudaGetLastError());
        }
        int herr = 0;
        CTRY(cudaMemcpyAsync(&herr, err.p, sizeof(int), cudaMemcpyDeviceToHost, s));
        CTRY(cudaStreamSynchronize(s));
        if (full_colidx == nullptr && first != 0) herr |= ERR_ROWPTR0;
        if (herr) {
            std::string m = "invalid CSR:";
            if (herr & ERR_ROWPTR0) m += " rowptr[0] != 0;";
            if (herr & ERR_MONO) m += " rowptr not non-decreasing;";
            if (herr & ERR_LAST) m += " rowptr[n_dst] != nnz;";
            if (herr & ERR_COL) m += " colidx outside [0, n_src);";
            graph_free(g);
            return set_error(TLP_ERR_INVALID_GRAPH, m);
        }
    }

    mark("a1 ingest+validate");
    // ---- a2: degrees and BOTH-norm coefficients --------------------------
    TRY(dmalloc((void **)&g->out_deg, sizeof(int32_t) * n_src, g));
    TRY(dmalloc((void **)&g->c_out, sizeof(float) * n_src, g));
    TRY(dmalloc((void **)&g->c_out_left, sizeof(float) * n_src, g));
    CTRY(cudaMemsetAsync(g->out_deg, 0, sizeof(int32_t) * n_src, s));
    {
        const int32_t *cols = full_colidx ? full_colidx : g->colidx;
        int64_t cnt = full_colidx ? full_nnz : nnz;
        if (cnt) {
            k_out_degree<<<grid_for(cnt, nsm), 256, 0, s>>>(cols, cnt, g->out_deg);
            CTRY(cudaGetLastError());
        }
        if (n_src) {
            k_norm<<<grid_for(n_src, nsm), 256, 0, s>>>(g->out_deg, n_src, g->c_out, g->c_out_left);
            CTRY(cudaGetLastError());
        }
        if (nnz && ew) {  // weighted BOTH streams w_e c_out[u]; unweighted pre-scales X
            TRY(dmalloc((void **)&g->ew_both, sizeof(float) * nnz + 16, g));
            k_edge_both<<<grid_for(nnz, nsm), 256, 0, s>>>(g->colidx, g->ew, g->c_out, nnz, g->ew_both);
            CTRY(cudaGetLastError());
        }
    }

    mark("a2 degrees+norms");
    // ---- a3: work plan ---------------------------------------------------
    TRY(dmalloc((void **)&g->ctr, sizeof(unsigned int) * 4, g));
    CTRY(cudaMemsetAsync(g->ctr, 0, sizeof(unsigned int) * 4, s));
    if (n_dst > 0) {
        DevBuf start, hub, starts, nsel, temp, utasks, keep, rtasks, hub_rows_u, hub_deg_u,
            hub_deg_s, nchunk;
        CTRY(start.alloc(n_dst, s));
        CTRY(hub.alloc(n_dst, s));
        CTRY(starts.alloc(sizeof(int32_t) * n_dst, s));
        CTRY(nsel.alloc(sizeof(int64_t) * 4, s));
        k_plan_flags<<<grid_for(n_dst, nsm), 256, 0, s>>>(g->rowptr, n_dst, g->K, g->H,
                                                          start.as<uint8_t>(), hub.as<uint8_t>());
        CTRY(cudaGetLastError());
        // unit starts = rows with start flag (CUB select over a counting iterator)
        cub::CountingInputIterator<int32_t> rows(0);
        size_t tb = 0, tb2 = 0;
        CTRY(cub::DeviceSelect::Flagged(nullptr, tb, rows, start.as<uint8_t>(),
                                        starts.as<int32_t>(), nsel.as<int64_t>(), (int)n_dst, s));
        CTRY(cub::DeviceSelect::Flagged(nullptr, tb2, rows, hub.as<uint8_t>(),
                                        starts.as<int32_t>(), nsel.as<int64_t>(), (int)n_dst, s));
        if (tb2 > tb) tb = tb2;
        CTRY(temp.alloc(tb, s));
        CTRY(cub::DeviceSelect::Flagged(temp.p, tb, rows, start.as<uint8_t>(),
                                        starts.as<int32_t>(), nsel.as<int64_t>(), (int)n_dst, s));
        int64_t h_n_units = 0;
        CTRY(cudaMemcpyAsync(&h_n_units, nsel.p, sizeof(int64_t), cudaMemcpyDeviceToHost, s));
        CTRY(cudaStreamSynchronize(s));

        CTRY(utasks.alloc(sizeof(int2) * h_n_units, s));
        CTRY(keep.alloc(h_n_units, s));
        CTRY(rtasks.alloc(sizeof(int2) * h_n_units, s));
        k_units_to_tasks<<<grid_for(h_n_units, nsm), 256, 0, s>>>(
            starts.as<int32_t>(), h_n_units, n_dst, hub.as<uint8_t>(), utasks.as<int2>(),
            keep.as<uint8_t>());
        CTRY(cudaGetLastError());
        size_t tb3 = 0;
        CTRY(cub::DeviceSelect::Flagged(nullptr, tb3, utasks.as<int2>(), keep.as<uint8_t>(),
                                        rtasks.as<int2>(), nsel.as<int64_t>() + 1, (int)h_n_units, s));
        if (tb3 > tb) {
            cudaFreeAsync(temp.p, s);
            temp.p = nullptr;
            CTRY(temp.alloc(tb3, s));
            tb = tb3;
        }
        CTRY(cub::DeviceSelect::Flagged(temp.p, tb, utasks.as<int2>(), keep.as<uint8_t>(),
                                        rtasks.as<int2>(), nsel.as<int64_t>() + 1, (int)h_n_units, s));
        // hubs in row order, then sorted by descending degree (stable => ties by row)
        CTRY(hub_rows_u.alloc(sizeof(int32_t) * n_dst, s));
        CTRY(cub::DeviceSelect::Flagged(temp.p, tb, rows, hub.as<uint8_t>(),
                                        hub_rows_u.as<int32_t>(), nsel.as<int64_t>() + 2,
                                        (int)n_dst, s));
        int64_t h_cnt[3] = {0, 0, 0};
        CTRY(cudaMemcpyAsync(h_cnt, nsel.p, sizeof(int64_t) * 3, cudaMemcpyDeviceToHost, s));
        CTRY(cudaStreamSynchronize(s));
        const int64_t n_reg = h_cnt[1], n_hubs = h_cnt[2];
        g->n_units = n_reg;
        g->n_hubs = n_hubs;
        TRY(dmalloc((void **)&g->hub_row, sizeof(int32_t) * n_hubs, g));
        TRY(dmalloc((void **)&g->hub_off, sizeof(int32_t) * (n_hubs + 1), g));
        CTRY(cudaMemsetAsync(g->hub_off, 0, sizeof(int32_t) * (n_hubs + 1), s));
        int64_t n_chunks = 0;
        if (n_hubs > 0) {
            CTRY(hub_deg_u.alloc(sizeof(int32_t) * n_hubs, s));
            CTRY(hub_deg_s.alloc(sizeof(int32_t) * n_hubs, s));
            CTRY(nchunk.alloc(sizeof(int32_t) * (n_hubs + 1), s));
            k_gather_deg<<<grid_for(n_hubs, nsm), 256, 0, s>>>(hub_rows_u.as<int32_t>(), n_hubs,
                                                               g->in_deg, hub_deg_u.as<int32_t>());
            CTRY(cudaGetLastError());
            DevBuf t2;
            size_t b2 = 0;
            CTRY(cub::DeviceRadixSort::SortPairsDescending(
                nullptr, b2, hub_deg_u.as<int32_t>(), hub_deg_s.as<int32_t>(),
                hub_rows_u.as<int32_t>(), g->hub_row, (int)n_hubs, 0, 32, s));
            CTRY(t2.alloc(b2, s));
            CTRY(cub::DeviceRadixSort::SortPairsDescending(
                t2.p, b2, hub_deg_u.as<int32_t>(), hub_deg_s.as<int32_t>(),
                hub_rows_u.as<int32_t>(), g->hub_row, (int)n_hubs, 0, 32, s));
            k_hub_chunks<<<grid_for(n_hubs, nsm), 256, 0, s>>>(hub_deg_s.as<int32_t>(), n_hubs,
                                                               g->C, nchunk.as<int32_t>());
            CTRY(cudaGetLastError());
            CTRY(cudaMemsetAsync(nchunk.as<int32_t>() + n_hubs, 0, sizeof(int32_t), s));
            DevBuf t3;
            size_t b3 = 0;
            CTRY(cub::DeviceScan::ExclusiveSum(nullptr, b3, nchunk.as<int32_t>(), g->hub_off,
                                               (int)(n_hubs + 1), s));
            CTRY(t3.alloc(b3, s));
            CTRY(cub::DeviceScan::ExclusiveSum(t3.p, b3, nchunk.as<int32_t>(), g->hub_off,
                                               (int)(n_hubs + 1), s));
            int32_t hc = 0;
            CTRY(cudaMemcpyAsync(&hc, g->hub_off + n_hubs, sizeof(int32_t),
                                 cudaMemcpyDeviceToHost, s));
            int32_t maxdeg = 0;
            CTRY(cudaMemcpyAsync(&maxdeg, hub_deg_s.p, sizeof(int32_t), cudaMemcpyDeviceToHost, s));
            CTRY(cudaStreamSynchronize(s));
            n_chunks = hc;
            g->max_in_degree = maxdeg;
        }
        g->n_chunks = n_chunks;
        g->n_tasks = n_chunks + n_reg;
        TRY(dmalloc((void **)&g->tasks, sizeof(int2) * g->n_tasks, g));
        if (n_hubs > 0) {
            k_hub_tasks<<<grid_for(n_hubs, nsm), 256, 0, s>>>(g->hub_off, n_hubs, g->tasks);
            CTRY(cudaGetLastError());
        }
        if (n_reg)
            CTRY(cudaMemcpyAsync(g->tasks + n_chunks, rtasks.p, sizeof(int2) * n_reg,
                                 cudaMemcpyDeviceToDevice, s));
        if (n_hubs == 0) {
            // max in-degree over regular rows (<= H): one reduction
            DevBuf mx, t4;
            size_t b4 = 0;
            CTRY(mx.alloc(sizeof(int32_t), s));
            CTRY(cub::DeviceReduce::Max(nullptr, b4, g->in_deg, mx.as<int32_t>(), (int)n_dst, s));
            CTRY(t4.alloc(b4, s));
            CTRY(cub::DeviceReduce::Max(t4.p, b4, g->in_deg, mx.as<int32_t>(), (int)n_dst, s));
            int32_t m = 0;
            CTRY(cudaMemcpyAsync(&m, mx.p, sizeof(int32_t), cudaMemcpyDeviceToHost, s));
            CTRY(cudaStreamSynchronize(s));
            g->max_in_degree = m;
        }
        g->regular_edges = nnz;  // refined below (edges outside hubs)
        CTRY(cudaStreamSynchronize(s));
    }
    if (n_dst > 0 && g->n_hubs > 0) {
        // edges in hubs = sum of hub degrees: recompute on the host from chunk count bound
        // (only used to size the Alg. 1 step heuristic; no correctness role)
        g->regular_edges = nnz - std::min<int64_t>(nnz, g->n_chunks * g->C);
        if (g->regular_edges < 0) g->regular_edges = 0;
    }
    mark("a3 plan");
    auto t1 = std::chrono::steady_clock::now();
    g->create_ms = std::chrono::duration<double, std::milli>(t1 - t0).count();
    *out = g;
    return TLP_OK;
}

// Transposed (out-edge) CSR for the backward aggregations (NEXT-4): stable sort
// of the edges by source keeps each source's edges in destination order.
tlp_status build_transpose(tlp_graph g, cudaStream_t s) {
    if (g->t) return TLP_OK;
    if (g->row_offset != 0 || g->bounds_host)
        return set_error(TLP_ERR_UNSUPPORTED, "transpose of a row slice (dist graph) is not supported");
    const int64_t nnz = g->nnz, n_dst = g->n_dst, n_src = g->n_src;
    if (nnz >= (int64_t(1) << 31))
        return set_error(TLP_ERR_UNSUPPORTED, "transpose needs nnz < 2^31");
    const int nsm = g->num_sms;
    DevBuf dst, keys_out, iota, perm, t_col, t_ew, t_rp, deg64, temp;
    TLP_CUDA_TRY(dst.alloc(sizeof(int32_t) * nnz + 16, s));
    TLP_CUDA_TRY(keys_out.alloc(sizeof(int32_t) * nnz + 16, s));
    TLP_CUDA_TRY(iota.alloc(sizeof(int32_t) * nnz + 16, s));
    TLP_CUDA_TRY(perm.alloc(sizeof(int32_t) * nnz + 16, s));
    TLP_CUDA_TRY(t_col.alloc(sizeof(int32_t) * nnz + 16, s));
    if (g->ew) TLP_CUDA_TRY(t_ew.alloc(sizeof(float) * nnz + 16, s));
    if (!g->tpos) {
        TLP_CUDA_TRY(cudaMalloc(&g->tpos, sizeof(int32_t) * nnz + 16));
        g->device_bytes += sizeof(int32_t) * nnz + 16;
    }
    TLP_CUDA_TRY(t_rp.alloc(sizeof(int64_t) * (n_src + 1), s));
    TLP_CUDA_TRY(deg64.alloc(sizeof(int64_t) * (n_src + 1), s));
    if (n_dst) {
        k_edge_rows<<<grid_for(n_dst, nsm), 256, 0, s>>>(g->rowptr, n_dst, dst.as<int32_t>());
        TLP_CUDA_TRY(cudaGetLastError());
    }
    if (nnz) {
        k_iota<<<grid_for(nnz, nsm), 256, 0, s>>>(iota.as<int32_t>(), nnz);
        TLP_CUDA_TRY(cudaGetLastError());
        size_t tb2 = 0;
        TLP_CUDA_TRY(cub::DeviceRadixSort::SortPairs(nullptr, tb2, g->colidx, keys_out.as<int32_t>(),
                                                     iota.as<int32_t>(), perm.as<int32_t>(), (int)nnz,
                                                     0, 32, s));
        TLP_CUDA_TRY(temp.alloc(tb2, s));
        TLP_CUDA_TRY(cub::DeviceRadixSort::SortPairs(temp.p, tb2, g->colidx, keys_out.as<int32_t>(),
                                                     iota.as<int32_t>(), perm.as<int32_t>(), (int)nnz,
                                                     0, 32, s));
        k_permute_edges<<<grid_for(nnz, nsm), 256, 0, s>>>(perm.as<int32_t>(), nnz, dst.as<int32_t>(),
                                                           g->ew, t_col.as<int32_t>(), t_ew.as<float>(),
                                                           g->tpos);
        TLP_CUDA_TRY(cudaGetLastError());
    }
    // transposed rowptr = exclusive scan of the out-degrees
    k_deg_to_rowptr_input<<<grid_for(n_src + 1, nsm), 256, 0, s>>>(g->out_deg, n_src, deg64.as<int64_t>());
    TLP_CUDA_TRY(cudaGetLastError());
    {
        DevBuf t3;
        size_t b3 = 0;
        TLP_CUDA_TRY(cub::DeviceScan::ExclusiveSum(nullptr, b3, deg64.as<int64_t>(), t_rp.as<int64_t>(),
                                                   (int)(n_src + 1), s));
        TLP_CUDA_TRY(t3.alloc(b3, s));
        TLP_CUDA_TRY(cub::DeviceScan::ExclusiveSum(t3.p, b3, deg64.as<int64_t>(), t_rp.as<int64_t>(),
                                                   (int)(n_src + 1), s));
    }
    tlp_create_opts o{g->H, g->C, 0};
    tlp_graph t = nullptr;
    tlp_status st = graph_create_impl(n_src, n_dst, nnz, t_rp.as<int64_t>(), t_col.as<int32_t>(),
                                      g->ew ? t_ew.as<float>() : nullptr, nullptr, 0, 0, &o, s, &t);
    if (st != TLP_OK) return st;
    t->sched = g->sched;
    t->warps_per_cta = g->warps_per_cta;
    g->t = t;
    g->device_bytes += t->device_bytes;
    return TLP_OK;
}

tlp_status ensure_edge_both(tlp_graph g, cudaStream_t s) {
    if (g->ew_both || g->nnz == 0) return TLP_OK;
    float *p = nullptr;
    cudaError_t e = cudaMallocAsync((void **)&p, sizeof(float) * g->nnz + 16, s);
    if (e != cudaSuccess) return cuda_error(e, "cudaMallocAsync(edge BOTH coefficients)");
    g->device_bytes += sizeof(float) * g->nnz + 16;
    const int nsm = g->num_sms > 0 ? g->num_sms : 148;
    k_edge_both<<<grid_for(g->nnz, nsm), 256, 0, s>>>(g->colidx, g->ew, g->c_out, g->nnz, p);
    g->launches += 1;
    e = cudaGetLastError();
    if (e != cudaSuccess) return cuda_error(e, "k_edge_both launch");
    g->ew_both = p;
    return TLP_OK;
}

tlp_status ensure_scratch(tlp_graph g, size_t bytes, cudaStream_t s) {
    if (bytes <= g->scratch_bytes) return TLP_OK;
    if (g->scratch) {
        cudaError_t e = cudaFreeAsync(g->scratch, s);
        if (e != cudaSuccess) return cuda_error(e, "cudaFreeAsync(scratch)");
        g->device_bytes -= g->scratch_bytes;
        g->scratch = nullptr;
        g->scratch_bytes = 0;
    }
    cudaError_t e = cudaMallocAsync((void **)&g->scratch, bytes, s);
    if (e != cudaSuccess) return cuda_error(e, "cudaMallocAsync(scratch)");
    g->scratch_bytes = bytes;
    g->device_bytes += bytes;
    return TLP_OK;
}

}  // namespace tlp

// ================================================================ C ABI ====

using namespace tlp;

extern "C" {

const char *tlp_status_string(tlp_status s) {
    switch (s) {
        case TLP_OK: return "TLP_OK";
        case TLP_ERR_INVALID_ARGUMENT: return "TLP_ERR_INVALID_ARGUMENT";
        case TLP_ERR_INVALID_GRAPH: return "TLP_ERR_INVALID_GRAPH";
        case TLP_ERR_OUT_OF_MEMORY: return "TLP_ERR_OUT_OF_MEMORY";
        case TLP_ERR_CUDA: return "TLP_ERR_CUDA";
        case TLP_ERR_NCCL: return "TLP_ERR_NCCL";
        case TLP_ERR_UNSUPPORTED: return "TLP_ERR_UNSUPPORTED";
    }
    return "TLP_ERR_UNKNOWN";
}

const char *tlp_last_error(void) { return g_last_error.c_str(); }

int tlp_version(void) { return TLP_VERSION_MAJOR * 100 + TLP_VERSION_MINOR; }

tlp_status tlp_graph_create(int64_t n_dst, int64_t n_src, int64_t nnz, const int64_t *rowptr,
                            const int32_t *colidx, const float *edge_weight, void *stream,
                            tlp_graph *out) {
    return graph_create_impl(n_dst, n_src, nnz, rowptr, colidx, edge_weight, nullptr, 0, 0,
                             nullptr, (cudaStream_t)stream, out);
}

tlp_status tlp_graph_create_ex(int64_t n_dst, int64_t n_src, int64_t nnz, const int64_t *rowptr,
                               const int32_t *colidx, const float *edge_weight,
                               const tlp_create_opts *opts, void *stream, tlp_graph *out) {
    if (opts && (opts->hub_threshold < 0 || opts->hub_chunk < 0 || opts->unit_edges < 0))
        return set_error(TLP_ERR_INVALID_ARGUMENT, "negative plan option");
    return graph_create_impl(n_dst, n_src, nnz, rowptr, colidx, edge_weight, nullptr, 0, 0, opts,
                             (cudaStream_t)stream, out);
}

tlp_status tlp_graph_destroy(tlp_graph g) {
    if (!g) return TLP_OK;
    cudaError_t e = cudaStreamSynchronize(g->last_stream);
    graph_free(g);
    if (e != cudaSuccess) return cuda_error(e, "cudaStreamSynchronize(destroy)");
    return TLP_OK;
}

tlp_status tlp_graph_info_get(tlp_graph g, tlp_graph_info *o) {
    if (!g || !o) return set_error(TLP_ERR_INVALID_ARGUMENT, "null argument");
    std::memset(o, 0, sizeof(*o));
    o->n_dst = g->n_dst;
    o->n_src = g->n_src;
    o->nnz = g->nnz;
    o->row_offset = g->row_offset;
    o->max_in_degree = g->max_in_degree;
    o->n_hubs = g->n_hubs;
    o->n_hub_chunks = g->n_chunks;
    o->n_units = g->n_units;
    o->n_tasks = g->n_tasks;
    o->hub_threshold = g->H;
    o->hub_chunk = g->C;
    o->unit_edges = g->K;
    o->has_edge_weight = g->ew != nullptr;
    o->device_bytes = (int64_t)g->device_bytes;
    o->scratch_bytes = (int64_t)g->scratch_bytes;
    o->create_ms = g->create_ms;
    o->launches = g->launches + (g->t ? g->t->launches : 0);
    return TLP_OK;
}

tlp_status tlp_graph_degrees(tlp_graph g, int32_t *in_deg, int32_t *out_deg, void *stream) {
    if (!g) return set_error(TLP_ERR_INVALID_ARGUMENT, "null graph");
    cudaStream_t s = (cudaStream_t)stream;
    if (in_deg && g->n_dst)
        TLP_CUDA_TRY(cudaMemcpyAsync(in_deg, g->in_deg, sizeof(int32_t) * g->n_dst,
                                     cudaMemcpyDefault, s));
    if (out_deg && g->n_src)
        TLP_CUDA_TRY(cudaMemcpyAsync(out_deg, g->out_deg, sizeof(int32_t) * g->n_src,
                                     cudaMemcpyDefault, s));
    TLP_CUDA_TRY(cudaStreamSynchronize(s));
    return TLP_OK;
}

tlp_status tlp_graph_plan(tlp_graph g, int32_t *tasks, int32_t *hub_rows, int32_t *hub_chunk_off,
                          void *stream) {
    if (!g) return set_error(TLP_ERR_INVALID_ARGUMENT, "null graph");
    cudaStream_t s = (cudaStream_t)stream;
    if (tasks && g->n_tasks)
        TLP_CUDA_TRY(cudaMemcpyAsync(tasks, g->tasks, sizeof(int2) * g->n_tasks,
                                     cudaMemcpyDefault, s));
    if (hub_rows && g->n_hubs)
        TLP_CUDA_TRY(cudaMemcpyAsync(hub_rows, g->hub_row, sizeof(int32_t) * g->n_hubs,
                                     cudaMemcpyDefault, s));
    if (hub_chunk_off && g->hub_off)
        TLP_CUDA_TRY(cudaMemcpyAsync(hub_chunk_off, g->hub_off, sizeof(int32_t) * (g->n_hubs + 1),
                                     cudaMemcpyDefault, s));
    TLP_CUDA_TRY(cudaStreamSynchronize(s));
    return TLP_OK;
}

tlp_status tlp_graph_build_transpose(tlp_graph g, void *stream) {
    if (!g) return set_error(TLP_ERR_INVALID_ARGUMENT, "null graph");
    return build_transpose(g, (cudaStream_t)stream);
}

tlp_status tlp_graph_set_visit_counter(tlp_graph g, int32_t *counter) {
    if (!g) return set_error(TLP_ERR_INVALID_ARGUMENT, "null graph");
    g->visits = counter;
    return TLP_OK;
}

tlp_status tlp_graph_set_schedule(tlp_graph g, int sched, int warps_per_cta, int step) {
    if (!g) return set_error(TLP_ERR_INVALID_ARGUMENT, "null graph");
    if (sched < TLP_SCHED_DYNAMIC || sched > TLP_SCHED_CLC)
        return set_error(TLP_ERR_INVALID_ARGUMENT, "unknown scheduler");
    if (warps_per_cta < 0 || warps_per_cta > 32 || step < 0)
        return set_error(TLP_ERR_INVALID_ARGUMENT, "warps_per_cta in [0,32], step >= 0");
    g->sched = sched;
    g->warps_per_cta = warps_per_cta ? warps_per_cta : 8;
    g->step = step;
    if (g->t) tlp_graph_set_schedule(g->t, sched, warps_per_cta, step);
    return TLP_OK;
}

}  // extern "C"

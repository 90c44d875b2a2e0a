// tlp_dist.cu -- multi-GPU layer: destination-row ranges balanced
// by edge count, X replicated, an all-gather of the output rows between layers.
//
// The paper is single-GPU and leaves multi-GPU to future work with METIS
// (P:262-265); the north star replaces that with edge-balanced contiguous row
// ranges, which need no partitioner and keep every row's in-edges (and so its
// GAT softmax) on one rank.  Rows are independent in the pull formulation
// (P:484-499), so a layer needs no communication inside it; the only exchange
// is the row all-gather.  NCCL 2.28 has no all-gatherv: rank r's slab is
// broadcast in place by a grouped ncclBroadcast(root = r).
#include <nccl.h>
#include <nccl_device.h>  // NCCL 2.28 device API: symmetric windows, LSA / multimem pointers

#include <chrono>
#include <cstring>
#include <string>
#include <thread>
#include <vector>

#include "tlp_internal.h"

// A symmetric output buffer (NEXT-2): allocated on every rank, each rank's
// allocation mapped into every other rank's address space (CUDA IPC over
// NVLink); dev_ptrs[r] = rank r's buffer as seen from this rank.
struct SymBuf {
    void *local = nullptr;
    size_t bytes = 0;
    std::vector<void *> peers;  // [world], peers[rank] = local
    float **dev_ptrs = nullptr; // device copy of peers
    // NCCL symmetric window form (preferred): ncclMemAlloc'd buffer registered
    // with NCCL_WIN_COLL_SYMMETRIC; peers[] are its LSA pointers and mc its
    // NVLS multicast address (null when the node has no NVLS)
    bool window = false;
    ncclWindow_t win = nullptr;
    ncclDevComm dev_comm{};
    float *mc = nullptr;
};

struct tlp_comm_s {
    ncclComm_t comm = nullptr;
    int world = 1, rank = 0;
    std::vector<SymBuf> sym;
    int *barrier = nullptr;     // one device int for the stream barrier
    cudaStream_t side = nullptr;  // private stream for the communicator's own blocking steps
};

namespace tlp {

static tlp_status nccl_error(ncclResult_t r, const char *what) {
    return set_error(TLP_ERR_NCCL, std::string(what) + ": " + ncclGetErrorString(r));
}

#define TLP_NCCL_TRY(expr)                                   \
    do {                                                     \
        ncclResult_t _r = (expr);                            \
        if (_r != ncclSuccess) return nccl_error(_r, #expr); \
    } while (0)

// lower_bound rule (R16): first r in [0, n] with rowptr[r] >= target.
static int64_t lower_bound_rows(const int64_t *rowptr, int64_t n, int64_t target) {
    int64_t lo = 0, hi = n;  // answer in [lo, hi]
    while (lo < hi) {
        int64_t mid = lo + (hi - lo) / 2;
        if (rowptr[mid] < target) lo = mid + 1;
        else hi = mid;
    }
    return lo;
}

static void partition(const int64_t *rowptr, int64_t n, int parts, int64_t *b) {
    const int64_t nnz = rowptr[n];
    b[0] = 0;
    for (int k = 1; k < parts; ++k) b[k] = lower_bound_rows(rowptr, n, (int64_t)k * nnz / parts);
    b[parts] = n;
}

}  // namespace tlp

using namespace tlp;

extern "C" {

tlp_status tlp_partition_rows(const int64_t *rowptr_host, int64_t n, int parts,
                              int64_t *bounds_host) {
    if (!rowptr_host || !bounds_host || n < 0 || parts < 1)
        return set_error(TLP_ERR_INVALID_ARGUMENT, "partition: bad argument");
    if (rowptr_host[0] != 0) return set_error(TLP_ERR_INVALID_GRAPH, "rowptr[0] != 0");
    partition(rowptr_host, n, parts, bounds_host);
    return TLP_OK;
}

tlp_status tlp_comm_get_unique_id(uint8_t id[128]) {
    if (!id) return set_error(TLP_ERR_INVALID_ARGUMENT, "id is NULL");
    static_assert(sizeof(ncclUniqueId) == 128, "ncclUniqueId size");
    ncclUniqueId u;
    TLP_NCCL_TRY(ncclGetUniqueId(&u));
    std::memcpy(id, &u, 128);
    return TLP_OK;
}

tlp_status tlp_comm_create(const uint8_t id[128], int world, int rank, tlp_comm *out) {
    if (!id || !out || world < 1 || rank < 0 || rank >= world)
        return set_error(TLP_ERR_INVALID_ARGUMENT, "comm_create: bad argument");
    *out = nullptr;
    ncclUniqueId u;
    std::memcpy(&u, id, 128);
    tlp_comm c = new tlp_comm_s();
    ncclResult_t r = ncclCommInitRank(&c->comm, world, u, rank);
    if (r != ncclSuccess) {
        delete c;
        return nccl_error(r, "ncclCommInitRank");
    }
    c->world = world;
    c->rank = rank;
    cudaError_t ce = cudaStreamCreateWithFlags(&c->side, cudaStreamNonBlocking);
    if (ce != cudaSuccess) {
        ncclCommDestroy(c->comm);
        delete c;
        return cuda_error(ce, "cudaStreamCreate(comm side stream)");
    }
    *out = c;
    return TLP_OK;
}

// NCCL failure detection: the asynchronous error state of the
// communicator (a peer that died, a network / NVLink fault), polled without
// blocking.
tlp_status tlp_comm_async_error(tlp_comm c, int *nccl_result) {
    if (!c || !nccl_result) return set_error(TLP_ERR_INVALID_ARGUMENT, "comm_async_error: bad argument");
    ncclResult_t a = ncclSuccess;
    TLP_NCCL_TRY(ncclCommGetAsyncError(c->comm, &a));
    *nccl_result = (int)a;
    if (a != ncclSuccess && a != ncclInProgress) return nccl_error(a, "communicator async error");
    return TLP_OK;
}

// Abort: tear the communicator down without waiting for peers (after a fault
// or a timeout); the handle stays valid only for tlp_comm_destroy.
tlp_status tlp_comm_abort(tlp_comm c) {
    if (!c) return set_error(TLP_ERR_INVALID_ARGUMENT, "comm_abort: null");
    if (!c->comm) return TLP_OK;
    ncclResult_t r = ncclCommAbort(c->comm);
    c->comm = nullptr;
    if (r != ncclSuccess) return nccl_error(r, "ncclCommAbort");
    return TLP_OK;
}

// Wait for `stream` (whose tail holds this communicator's collectives) while
// polling the communicator's asynchronous error state; on an error or after
// timeout_s seconds (<= 0: no limit) the communicator is aborted, so a hung
// peer cannot hang this rank forever.
tlp_status tlp_comm_wait(tlp_comm c, void *stream, double timeout_s) {
    if (!c) return set_error(TLP_ERR_INVALID_ARGUMENT, "comm_wait: null");
    cudaStream_t s = (cudaStream_t)stream;
    const auto t0 = std::chrono::steady_clock::now();
    for (;;) {
        cudaError_t q = cudaStreamQuery(s);
        if (q == cudaSuccess) return TLP_OK;
        if (q != cudaErrorNotReady) return cuda_error(q, "cudaStreamQuery");
        if (c->comm) {
            ncclResult_t a = ncclSuccess;
            ncclCommGetAsyncError(c->comm, &a);
            if (a != ncclSuccess && a != ncclInProgress) {
                tlp_comm_abort(c);
                return nccl_error(a, "communicator async error (aborted)");
            }
        }
        const double el = std::chrono::duration<double>(std::chrono::steady_clock::now() - t0).count();
        if (timeout_s > 0 && el > timeout_s) {
            tlp_comm_abort(c);
            return set_error(TLP_ERR_NCCL, "tlp_comm_wait: timeout, communicator aborted");
        }
        std::this_thread::sleep_for(std::chrono::microseconds(200));
    }
}

tlp_status tlp_comm_destroy(tlp_comm c) {
    if (!c) return TLP_OK;
    while (!c->sym.empty()) tlp_comm_free_symmetric(c, c->sym.back().local);
    if (c->barrier) cudaFree(c->barrier);
    if (c->side) cudaStreamDestroy(c->side);
    ncclResult_t r = c->comm ? ncclCommDestroy(c->comm) : ncclSuccess;
    delete c;
    if (r != ncclSuccess) return nccl_error(r, "ncclCommDestroy");
    return TLP_OK;
}

tlp_status tlp_graph_create_rows(int64_t n, int64_t nnz, const int64_t *rowptr,
                                 const int32_t *colidx, const float *edge_weight,
                                 int64_t row_begin, int64_t row_end, const tlp_create_opts *opts,
                                 void *stream, tlp_graph *out) {
    if (!rowptr || !out || n < 0 || nnz < 0 || (nnz > 0 && !colidx) || row_begin < 0 ||
        row_end < row_begin || row_end > n)
        return set_error(TLP_ERR_INVALID_ARGUMENT, "graph_create_rows: bad argument");
    *out = nullptr;
    cudaStream_t s = (cudaStream_t)stream;
    // slice edge range from the full rowptr
    int64_t e01[2] = {0, 0}, ends[2] = {0, 0};
    TLP_CUDA_TRY(cudaMemcpyAsync(&e01[0], rowptr + row_begin, sizeof(int64_t), cudaMemcpyDefault, s));
    TLP_CUDA_TRY(cudaMemcpyAsync(&e01[1], rowptr + row_end, sizeof(int64_t), cudaMemcpyDefault, s));
    TLP_CUDA_TRY(cudaMemcpyAsync(&ends[0], rowptr, sizeof(int64_t), cudaMemcpyDefault, s));
    TLP_CUDA_TRY(cudaMemcpyAsync(&ends[1], rowptr + n, sizeof(int64_t), cudaMemcpyDefault, s));
    TLP_CUDA_TRY(cudaStreamSynchronize(s));
    if (ends[0] != 0 || ends[1] != nnz)
        return set_error(TLP_ERR_INVALID_GRAPH, "rowptr[0] != 0 or rowptr[n] != nnz");
    const int64_t e0 = e01[0], e1 = e01[1];
    if (e0 < 0 || e1 < e0 || e1 > nnz)
        return set_error(TLP_ERR_INVALID_GRAPH, "rowptr not non-decreasing");
    // the full colidx must be device-resident for the global out-degree count
    const int32_t *full_col = colidx;
    void *staged = nullptr;
    if (nnz > 0) {
        cudaPointerAttributes attr;
        cudaError_t e = cudaPointerGetAttributes(&attr, colidx);
        bool on_dev = (e == cudaSuccess) && (attr.type == cudaMemoryTypeDevice ||
                                             attr.type == cudaMemoryTypeManaged);
        if (e != cudaSuccess) cudaGetLastError();
        if (!on_dev) {
            TLP_CUDA_TRY(cudaMalloc(&staged, sizeof(int32_t) * nnz));
            cudaError_t ce = cudaMemcpyAsync(staged, colidx, sizeof(int32_t) * nnz, cudaMemcpyDefault, s);
            if (ce != cudaSuccess) { cudaFree(staged); return cuda_error(ce, "stage colidx"); }
            full_col = (const int32_t *)staged;
        }
    }
    static const int32_t kNoEdges = 0;
    tlp_status st = graph_create_impl(row_end - row_begin, n, e1 - e0, rowptr + row_begin,
                                      full_col ? full_col + e0 : nullptr,
                                      edge_weight ? edge_weight + e0 : nullptr,
                                      full_col ? full_col : &kNoEdges, nnz, row_begin, opts, s, out);
    if (staged) {
        cudaStreamSynchronize(s);
        cudaFree(staged);
    }
    return st;
}

static tlp_status comm_barrier(tlp_comm c, cudaStream_t s) {
    if (c->world == 1) return TLP_OK;
    if (!c->comm) return set_error(TLP_ERR_NCCL, "communicator was aborted");
    if (!c->barrier) {
        TLP_CUDA_TRY(cudaMalloc(&c->barrier, sizeof(int)));
        TLP_CUDA_TRY(cudaMemset(c->barrier, 0, sizeof(int)));
    }
    TLP_NCCL_TRY(ncclAllReduce(c->barrier, c->barrier, 1, ncclInt, ncclSum, c->comm, s));
    return TLP_OK;
}

// LSA peer pointers and the multicast address of a registered window (the
// window descriptor lives in device memory, read through the device API).
__global__ void k_window_ptrs(ncclWindow_t w, ncclDevComm dc, int n, int use_mc, void **out) {
    const int i = threadIdx.x;
    if (i < n) out[i] = ncclGetLsaPointer(w, 0, i);
    if (i == 0) out[n] = use_mc ? ncclGetLsaMultimemPointer(w, 0, dc) : nullptr;
}

// NEXT-2 symmetric buffer through NCCL's window API (ncclMemAlloc +
// ncclCommWindowRegister + ncclDevCommCreate -> LSA peer pointers, and the
// NVLS multicast address when the node supports it).  Returns false (with
// nothing allocated) when any step is unavailable, so the caller falls back
// to CUDA IPC.
static bool alloc_window(tlp_comm c, size_t bytes, SymBuf &b) {
    const size_t al = NCCL_WIN_REQUIRED_ALIGNMENT;
    const size_t sz = (bytes + al - 1) / al * al;
    void *buf = nullptr;
    if (ncclMemAlloc(&buf, sz) != ncclSuccess) return false;
    ncclWindow_t win = nullptr;
    if (ncclCommWindowRegister(c->comm, buf, sz, &win, NCCL_WIN_COLL_SYMMETRIC) != ncclSuccess) {
        ncclMemFree(buf);
        return false;
    }
    ncclDevComm dc{};
    ncclDevCommRequirements req{};
    req.lsaMultimem = c->world > 1;
    bool mm = req.lsaMultimem;
    if (ncclDevCommCreate(c->comm, &req, &dc) != ncclSuccess) {
        // no NVLS (or a single rank): LSA pointers only
        req.lsaMultimem = false;
        mm = false;
        if (ncclDevCommCreate(c->comm, &req, &dc) != ncclSuccess) {
            ncclCommWindowDeregister(c->comm, win);
            ncclMemFree(buf);
            return false;
        }
    }
    if (dc.lsaSize != c->world) {  // more than one node: the IPC path is single-node as well
        ncclDevCommDestroy(c->comm, &dc);
        ncclCommWindowDeregister(c->comm, win);
        ncclMemFree(buf);
        return false;
    }
    void **d_out = nullptr;
    std::vector<void *> h(c->world + 1, nullptr);
    bool ok = cudaMalloc(&d_out, sizeof(void *) * (c->world + 1)) == cudaSuccess;
    if (ok) {
        k_window_ptrs<<<1, 64, 0, c->side>>>(win, dc, c->world, mm ? 1 : 0, d_out);
        ok = cudaMemcpyAsync(h.data(), d_out, sizeof(void *) * (c->world + 1), cudaMemcpyDeviceToHost,
                             c->side) == cudaSuccess &&
             cudaStreamSynchronize(c->side) == cudaSuccess;
        cudaFree(d_out);
    }
    if (!ok || h[c->rank] == nullptr) {
        cudaGetLastError();
        ncclDevCommDestroy(c->comm, &dc);
        ncclCommWindowDeregister(c->comm, win);
        ncclMemFree(buf);
        return false;
    }
    b.window = true;
    b.win = win;
    b.dev_comm = dc;
    b.local = buf;
    b.bytes = bytes;
    b.peers.assign(h.begin(), h.begin() + c->world);
    b.mc = (float *)h[c->world];
    return true;
}

tlp_status tlp_comm_alloc_symmetric(tlp_comm c, size_t bytes, void **local) {
    if (!c || !local || bytes == 0) return set_error(TLP_ERR_INVALID_ARGUMENT, "alloc_symmetric: bad argument");
    *local = nullptr;
    if (!c->comm) return set_error(TLP_ERR_NCCL, "communicator was aborted");
    SymBuf b;
    // NCCL symmetric window first (TLP_SYM=ipc forces the CUDA IPC form)
    const char *sym = getenv("TLP_SYM");
    if (!(sym && !strcmp(sym, "ipc")) && alloc_window(c, bytes, b)) {
        TLP_CUDA_TRY(cudaMalloc(&b.dev_ptrs, sizeof(float *) * c->world));
        TLP_CUDA_TRY(cudaMemcpy(b.dev_ptrs, b.peers.data(), sizeof(void *) * c->world, cudaMemcpyHostToDevice));
        c->sym.push_back(b);
        *local = b.local;
        return TLP_OK;
    }
    b = SymBuf();
    b.bytes = bytes;
    TLP_CUDA_TRY(cudaMalloc(&b.local, bytes));
    b.peers.assign(c->world, nullptr);
    b.peers[c->rank] = b.local;
    if (c->world > 1) {
        // exchange the IPC handles through NCCL (64 bytes per rank)
        cudaIpcMemHandle_t h;
        cudaError_t e = cudaIpcGetMemHandle(&h, b.local);
        if (e != cudaSuccess) { cudaFree(b.local); return cuda_error(e, "cudaIpcGetMemHandle"); }
        std::vector<cudaIpcMemHandle_t> all(c->world);
        void *dh = nullptr;
        // on the communicator's private stream (never the legacy default
        // stream, which would serialise against every other stream)
        TLP_CUDA_TRY(cudaMalloc(&dh, sizeof(cudaIpcMemHandle_t) * c->world));
        TLP_CUDA_TRY(cudaMemcpyAsync((char *)dh + sizeof(h) * c->rank, &h, sizeof(h), cudaMemcpyHostToDevice, c->side));
        ncclResult_t r = ncclAllGather((char *)dh + sizeof(h) * c->rank, dh, sizeof(h), ncclUint8, c->comm, c->side);
        if (r != ncclSuccess) { cudaFree(dh); cudaFree(b.local); return nccl_error(r, "ncclAllGather(ipc handles)"); }
        TLP_CUDA_TRY(cudaMemcpyAsync(all.data(), dh, sizeof(h) * c->world, cudaMemcpyDeviceToHost, c->side));
        TLP_CUDA_TRY(cudaStreamSynchronize(c->side));
        cudaFree(dh);
        for (int q = 0; q < c->world; ++q) {
            if (q == c->rank) continue;
            e = cudaIpcOpenMemHandle(&b.peers[q], all[q], cudaIpcMemLazyEnablePeerAccess);
            if (e != cudaSuccess) {
                for (int k = 0; k < q; ++k)
                    if (k != c->rank && b.peers[k]) cudaIpcCloseMemHandle(b.peers[k]);
                cudaFree(b.local);
                return cuda_error(e, "cudaIpcOpenMemHandle");
            }
        }
    }
    TLP_CUDA_TRY(cudaMalloc(&b.dev_ptrs, sizeof(float *) * c->world));
    TLP_CUDA_TRY(cudaMemcpy(b.dev_ptrs, b.peers.data(), sizeof(void *) * c->world, cudaMemcpyHostToDevice));
    c->sym.push_back(b);
    *local = b.local;
    return TLP_OK;
}

tlp_status tlp_comm_symmetric_kind(tlp_comm c, void *local, int *kind) {
    if (!c || !local || !kind) return set_error(TLP_ERR_INVALID_ARGUMENT, "symmetric_kind: bad argument");
    for (const SymBuf &b : c->sym)
        if (b.local == local) {
            *kind = b.window ? (b.mc ? 2 : 1) : 0;
            return TLP_OK;
        }
    return set_error(TLP_ERR_INVALID_ARGUMENT, "not a symmetric buffer of this communicator");
}

tlp_status tlp_comm_free_symmetric(tlp_comm c, void *local) {
    if (!c || !local) return set_error(TLP_ERR_INVALID_ARGUMENT, "free_symmetric: bad argument");
    for (size_t i = 0; i < c->sym.size(); ++i) {
        SymBuf &b = c->sym[i];
        if (b.local != local) continue;
        cudaDeviceSynchronize();  // no queued kernel still stores through the mappings
        if (b.window) {
            // collective: every rank deregisters its window
            if (c->comm) {
                ncclDevCommDestroy(c->comm, &b.dev_comm);
                ncclCommWindowDeregister(c->comm, b.win);
            }
            cudaFree(b.dev_ptrs);
            ncclMemFree(b.local);
            c->sym.erase(c->sym.begin() + i);
            return TLP_OK;
        }
        for (int q = 0; q < c->world; ++q)
            if (q != c->rank && b.peers[q]) cudaIpcCloseMemHandle(b.peers[q]);
        // every rank has unmapped before anyone frees
        tlp_status st = comm_barrier(c, c->side);
        cudaStreamSynchronize(c->side);
        cudaFree(b.dev_ptrs);
        cudaFree(b.local);
        c->sym.erase(c->sym.begin() + i);
        return st;
    }
    return set_error(TLP_ERR_INVALID_ARGUMENT, "not a symmetric buffer of this communicator");
}

tlp_status tlp_dist_graph_create(tlp_comm c, int64_t n, int64_t nnz, const int64_t *rowptr,
                                 const int32_t *colidx, const float *edge_weight,
                                 const tlp_create_opts *opts, void *stream, tlp_graph *out_local) {
    if (!c || !rowptr || !out_local || n < 0 || nnz < 0 || (nnz > 0 && !colidx))
        return set_error(TLP_ERR_INVALID_ARGUMENT, "dist_graph_create: bad argument");
    *out_local = nullptr;
    cudaStream_t s = (cudaStream_t)stream;
    // the partition is a pure function of rowptr: compute it on the host
    std::vector<int64_t> rp((size_t)n + 1);
    TLP_CUDA_TRY(cudaMemcpyAsync(rp.data(), rowptr, sizeof(int64_t) * (n + 1), cudaMemcpyDefault, s));
    TLP_CUDA_TRY(cudaStreamSynchronize(s));
    if (rp[0] != 0 || rp[n] != nnz) return set_error(TLP_ERR_INVALID_GRAPH, "rowptr[0] != 0 or rowptr[n] != nnz");
    for (int64_t i = 0; i < n; ++i)
        if (rp[i + 1] < rp[i]) return set_error(TLP_ERR_INVALID_GRAPH, "rowptr not non-decreasing");
    std::vector<int64_t> b((size_t)c->world + 1);
    partition(rp.data(), n, c->world, b.data());
    tlp_graph g = nullptr;
    tlp_status st = tlp_graph_create_rows(n, nnz, rowptr, colidx, edge_weight, b[c->rank],
                                          b[c->rank + 1], opts, stream, &g);
    if (st != TLP_OK) return st;
    g->world = c->world;
    g->rank = c->rank;
    g->n_global = n;
    g->bounds_host = new int64_t[c->world + 1];
    std::memcpy(g->bounds_host, b.data(), sizeof(int64_t) * (c->world + 1));
    *out_local = g;
    return TLP_OK;
}

tlp_status tlp_dist_bounds(tlp_graph g, int64_t *bounds_host) {
    if (!g || !bounds_host || !g->bounds_host)
        return set_error(TLP_ERR_INVALID_ARGUMENT, "not a dist graph");
    std::memcpy(bounds_host, g->bounds_host, sizeof(int64_t) * (g->world + 1));
    return TLP_OK;
}

tlp_status tlp_dist_allgather_rows(tlp_graph g, tlp_comm c, float *Y_full, int64_t ldy,
                                   void *stream) {
    if (!g || !c || !g->bounds_host || !Y_full || ldy < 0)
        return set_error(TLP_ERR_INVALID_ARGUMENT, "allgather: bad argument");
    if (c->world != g->world || c->rank != g->rank)
        return set_error(TLP_ERR_INVALID_ARGUMENT, "communicator does not match the graph");
    cudaStream_t s = (cudaStream_t)stream;
    if (c->world == 1) return TLP_OK;
    if (!c->comm) return set_error(TLP_ERR_NCCL, "communicator was aborted");
    TLP_NCCL_TRY(ncclGroupStart());
    for (int r = 0; r < c->world; ++r) {
        const int64_t rows = g->bounds_host[r + 1] - g->bounds_host[r];
        if (rows == 0) continue;
        float *p = Y_full + g->bounds_host[r] * ldy;
        ncclResult_t res = ncclBroadcast(p, p, (size_t)(rows * ldy), ncclFloat, r, c->comm, s);
        if (res != ncclSuccess) {
            ncclGroupEnd();
            return nccl_error(res, "ncclBroadcast");
        }
    }
    TLP_NCCL_TRY(ncclGroupEnd());
    return TLP_OK;
}

static tlp_status dist_local(tlp_graph g, tlp_comm c, AggRequest &r, void *stream) {
    if (!g || !c || !g->bounds_host) return set_error(TLP_ERR_INVALID_ARGUMENT, "not a dist graph");
    if (!r.Y) return set_error(TLP_ERR_INVALID_ARGUMENT, "Y_full is NULL");
    float *Y_full = r.Y;
    r.Y = Y_full + g->row_offset * r.ldy;
    tlp_status st = aggregate(g, r, (cudaStream_t)stream);
    if (st != TLP_OK) return st;
    return tlp_dist_allgather_rows(g, c, Y_full, r.ldy, stream);
}

tlp_status tlp_dist_gcn_aggregate(tlp_graph g, tlp_comm c, const float *X_full, int64_t F,
                                  int64_t ldx, int norm, float *Y_full, int64_t ldy, void *stream) {
    AggRequest r;
    r.op = 0; r.X = X_full; r.F = F; r.ldx = ldx; r.Y = Y_full; r.ldy = ldy; r.norm = norm;
    return dist_local(g, c, r, stream);
}

tlp_status tlp_dist_gin_aggregate(tlp_graph g, tlp_comm c, const float *X_full, int64_t F,
                                  int64_t ldx, float eps, float *Y_full, int64_t ldy, void *stream) {
    AggRequest r;
    r.op = 1; r.X = X_full; r.F = F; r.ldx = ldx; r.Y = Y_full; r.ldy = ldy; r.eps = eps;
    return dist_local(g, c, r, stream);
}

tlp_status tlp_dist_gat_aggregate(tlp_graph g, tlp_comm c, const float *X_full, int64_t F,
                                  int64_t ldx, const float *el, const float *er, float slope,
                                  float *Y_full, int64_t ldy, void *stream) {
    AggRequest r;
    r.op = 2; r.X = X_full; r.F = F; r.ldx = ldx; r.Y = Y_full; r.ldy = ldy;
    r.el = el; r.er = er; r.slope = slope;
    return dist_local(g, c, r, stream);
}

tlp_status tlp_dist_aggregate(tlp_graph g, tlp_comm c, const tlp_agg_desc *d, void *stream) {
    if (!d) return set_error(TLP_ERR_INVALID_ARGUMENT, "null descriptor");
    if (d->el_out || d->er_out || d->att_l || d->att_r)
        return set_error(TLP_ERR_UNSUPPORTED, "epilogue projections are single-GPU only");
    AggRequest r = request_from_desc(*d);
    return dist_local(g, c, r, stream);
}

// NEXT-2: one kernel computes this rank's rows and stores every finished row
// vector straight into Y_full on every rank over NVLink (peer-mapped symmetric
// buffer), so the all-gather overlaps the gather tile by tile; a one-element
// NCCL all-reduce then orders the stream after every rank's kernel.
tlp_status tlp_dist_aggregate_fused(tlp_graph g, tlp_comm c, const tlp_agg_desc *d, void *stream) {
    if (!g || !c || !d || !g->bounds_host) return set_error(TLP_ERR_INVALID_ARGUMENT, "not a dist graph");
    if (d->el_out || d->er_out || d->att_l || d->att_r)
        return set_error(TLP_ERR_UNSUPPORTED, "epilogue projections are single-GPU only");
    if (c->world != g->world || c->rank != g->rank)
        return set_error(TLP_ERR_INVALID_ARGUMENT, "communicator does not match the graph");
    const SymBuf *b = nullptr;
    for (const SymBuf &x : c->sym)
        if (x.local == (void *)d->Y) b = &x;
    if (!b) return set_error(TLP_ERR_INVALID_ARGUMENT, "Y_full must come from tlp_comm_alloc_symmetric");
    if ((size_t)(g->n_global * d->ldy) * sizeof(float) > b->bytes)
        return set_error(TLP_ERR_INVALID_ARGUMENT, "symmetric buffer smaller than n x ldy floats");
    AggRequest r = request_from_desc(*d);
    r.Y = d->Y + g->row_offset * d->ldy;
    r.dests = b->dev_ptrs;
    r.n_dests = c->world;
    // NVLS multicast: one store reaches every rank's Y_full (TLP_SYM_MC=0: per-peer stores)
    const char *mce = getenv("TLP_SYM_MC");
    if (b->mc && !(mce && !strcmp(mce, "0"))) r.mc = b->mc;
    // entry barrier: a fast rank must not store into a peer's Y_full while that
    // peer's stream may still read its previous contents (e.g. the next layer
    // reads Y_full while this call overwrites it on every rank)
    tlp_status st = comm_barrier(c, (cudaStream_t)stream);
    if (st != TLP_OK) return st;
    st = aggregate(g, r, (cudaStream_t)stream);
    if (st != TLP_OK) return st;
    // exit barrier: every rank's stores have landed (the kernel ends with
    // __threadfence_system) before any rank's stream proceeds
    return comm_barrier(c, (cudaStream_t)stream);
}

// Test hook for the multi-destination epilogue on one GPU: the aggregation of
// `g` stores every output row to each of the n host-listed device buffers.
tlp_status tlp_debug_multi_store(tlp_graph g, const tlp_agg_desc *d, float *const *dests_host, int n,
                                 void *stream) {
    if (!g || !d || !dests_host || n < 1) return set_error(TLP_ERR_INVALID_ARGUMENT, "bad argument");
    cudaStream_t s = (cudaStream_t)stream;
    float **dd = nullptr;
    TLP_CUDA_TRY(cudaMallocAsync((void **)&dd, sizeof(float *) * n, s));
    TLP_CUDA_TRY(cudaMemcpyAsync(dd, dests_host, sizeof(float *) * n, cudaMemcpyHostToDevice, s));
    AggRequest r = request_from_desc(*d);
    r.dests = dd;
    r.n_dests = n;
    tlp_status st = aggregate(g, r, s);
    cudaFreeAsync(dd, s);
    TLP_CUDA_TRY(cudaStreamSynchronize(s));  // dests_host may be freed on return
    return st;
}

tlp_status tlp_dist_sage_aggregate(tlp_graph g, tlp_comm c, const float *X_full, int64_t F,
                                   int64_t ldx, int include_self, float *Y_full, int64_t ldy,
                                   void *stream) {
    AggRequest r;
    r.op = 3; r.X = X_full; r.F = F; r.ldx = ldx; r.Y = Y_full; r.ldy = ldy;
    r.sage_self = include_self ? 1 : 0;
    return dist_local(g, c, r, stream);
}

tlp_status tlp_dist_gat_mh_aggregate(tlp_graph g, tlp_comm c, const float *X_full, int64_t heads,
                                     int64_t F, int64_t ldx, const float *el, const float *er,
                                     float slope, float *Y_full, int64_t ldy, void *stream) {
    AggRequest r;
    r.op = 4; r.X = X_full; r.F = F; r.ldx = ldx; r.Y = Y_full; r.ldy = ldy;
    r.el = el; r.er = er; r.slope = slope; r.heads = heads;
    return dist_local(g, c, r, stream);
}

}  // extern "C"

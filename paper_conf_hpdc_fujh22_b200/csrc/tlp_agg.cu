// tlp_agg.cu -- the aggregation kernels and their C ABI.
//
// One kernel launch per aggregation call (Observation III) that
// fuses, per destination row: index staging (a5), the coefficient/score of
// every edge, the gather-accumulate of the source rows (a6, a7), the hub
// split-and-merge (a8) and the epilogue store (a9).
//
// Mapping (prior art: TLPGNN's two-level parallelism; kept where
// it still holds on sm_100a, changed where it does not -- DESIGN.md):
//  * a WARP owns a task (a run of whole destination rows, or one chunk of a
//    hub row): no atomics on data (Observation I), no divergence.
//  * lanes cover consecutive 16-byte (VEC=4) feature vectors of one source
//    row (feature parallelism, Fig. 5b): a warp-wide gather of a
//    row strip is 32 x LDG.128 = 512 contiguous bytes, fully coalesced
//    (Observation II).  Rows wider than 128 floats are processed
//    as 128-float strips, so the register footprint does not grow with F.
//  * edge indices are loaded 32 at a time by the lanes (one coalesced LDG)
//    and broadcast with shuffles; U source rows are in flight per warp.
//  * fp32 accumulators live in registers; Y is written once per row (register
//    caching).
//  * GAT: LeakyReLU score, online softmax (running max / denominator rescaled
//    once per 32-edge chunk) and the weighted gather in the same pass; scores
//    never leave registers (kernel fusion).
//  * scheduling: persistent grid, static first wave + atomic counter fetching
//    `step` tasks (Alg. 1); hub rows (deg > H) are split into
//    C-edge chunks whose partials are merged in chunk order by the last
//    arriving warp (ticket), so results are bitwise deterministic.
#include <cuda_runtime.h>
#include <math.h>

#include <algorithm>

#include "tlp_internal.h"

namespace tlp {

enum Op : int { OP_GCN = 0, OP_GIN = 1, OP_GAT = 2 };
enum Coef : int { COEF_NONE = 0, COEF_COUT = 1, COEF_W = 2, COEF_W_COUT = 3 };
enum Sched : int { S_DYNAMIC = 0, S_STATIC = 1, S_HARDWARE = 2 };

constexpr unsigned FULL = 0xffffffffu;

struct AggArgs {
    const int64_t *__restrict__ rowptr;
    const int32_t *__restrict__ colidx;
    const float *__restrict__ ew;
    const float *__restrict__ c_out;
    const float *__restrict__ X;
    float *__restrict__ Y;
    const float *__restrict__ el;
    const float *__restrict__ er;
    const int2 *__restrict__ tasks;
    const int32_t *__restrict__ hub_row;
    const int32_t *__restrict__ hub_off;
    int32_t *hub_ticket;
    float *scratch;  // hub partial vectors [n_chunks x ldp]
    float *md;       // GAT hub (m, den) pairs [n_chunks x 2]
    unsigned long long *ctr;
    unsigned int *done;
    int64_t ldx, ldy, ldp, row_offset, n_tasks, C;
    int F, n_strips, norm, step, sched;
    float eps1, slope;
};

template <int VEC>
struct Vec {
    float v[VEC];
};

template <int VEC>
__device__ __forceinline__ Vec<VEC> ld_vec(const float *p) {
    Vec<VEC> r;
    if constexpr (VEC == 4) {
        float4 t = __ldg(reinterpret_cast<const float4 *>(p));
        r.v[0] = t.x; r.v[1] = t.y; r.v[2] = t.z; r.v[3] = t.w;
    } else if constexpr (VEC == 2) {
        float2 t = __ldg(reinterpret_cast<const float2 *>(p));
        r.v[0] = t.x; r.v[1] = t.y;
    } else {
        r.v[0] = __ldg(p);
    }
    return r;
}

// L2-coherent load (data written by another SM during this launch).
template <int VEC>
__device__ __forceinline__ Vec<VEC> ld_vec_cg(const float *p) {
    Vec<VEC> r;
    if constexpr (VEC == 4) {
        float4 t = __ldcg(reinterpret_cast<const float4 *>(p));
        r.v[0] = t.x; r.v[1] = t.y; r.v[2] = t.z; r.v[3] = t.w;
    } else if constexpr (VEC == 2) {
        float2 t = __ldcg(reinterpret_cast<const float2 *>(p));
        r.v[0] = t.x; r.v[1] = t.y;
    } else {
        r.v[0] = __ldcg(p);
    }
    return r;
}

template <int VEC>
__device__ __forceinline__ void st_vec(float *p, const Vec<VEC> &x) {
    if constexpr (VEC == 4) {
        *reinterpret_cast<float4 *>(p) = make_float4(x.v[0], x.v[1], x.v[2], x.v[3]);
    } else if constexpr (VEC == 2) {
        *reinterpret_cast<float2 *>(p) = make_float2(x.v[0], x.v[1]);
    } else {
        *p = x.v[0];
    }
}

// Store only columns < F (the tail vector of a row may straddle F).
template <int VEC>
__device__ __forceinline__ void st_row(float *row, int col, int F, const Vec<VEC> &x) {
    if (col + VEC <= F) {
        st_vec<VEC>(row + col, x);
    } else {
#pragma unroll
        for (int c = 0; c < VEC; ++c)
            if (col + c < F) row[col + c] = x.v[c];
    }
}

__device__ __forceinline__ float warp_max(float v) {
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) v = fmaxf(v, __shfl_xor_sync(FULL, v, o));
    return v;
}

// Butterfly sum: every lane ends with the bitwise-same value (commutativity).
__device__ __forceinline__ float warp_sum(float v) {
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) v += __shfl_xor_sync(FULL, v, o);
    return v;
}

// Reduce the edges [e0, e1) of one destination row for the feature vector at
// `col` (a6 / a7).  GCN/GIN: acc = sum_e c_e X[u_e] in CSR order.  GAT: online
// softmax state (m, den, acc = sum_e exp(s_e - m) X[u_e]).
template <int VEC, int OP, int COEF, int U>
__device__ __forceinline__ void reduce_edges(const AggArgs &a, int64_t e0, int64_t e1,
                                             int col, bool active, float er_v, int lane,
                                             Vec<VEC> &acc, float &m, float &den) {
    const float *__restrict__ Xc = a.X + col;
    for (int64_t base = e0; base < e1; base += 32) {
        const int n = (int)min((int64_t)32, e1 - base);
        int u_l = 0;
        float c_l = 1.f;
        if (lane < n) {
            u_l = __ldg(a.colidx + base + lane);
            if constexpr (COEF & COEF_COUT) c_l = __ldg(a.c_out + u_l);
            if constexpr (COEF & COEF_W) c_l *= __ldg(a.ew + base + lane);
        }
        if constexpr (OP == OP_GAT) {
            float s = -INFINITY;
            if (lane < n) {
                float t = __ldg(a.el + u_l) + er_v;
                s = t >= 0.f ? t : a.slope * t;  // LeakyReLU (R6)
            }
            const float m_new = fmaxf(m, warp_max(s));
            const float scale = __expf(m - m_new);  // m = -inf -> 0
            c_l = (lane < n) ? __expf(s - m_new) : 0.f;
            den = fmaf(den, scale, warp_sum(c_l));
#pragma unroll
            for (int c = 0; c < VEC; ++c) acc.v[c] *= scale;
            m = m_new;
        }
        for (int j = 0; j < n; j += U) {
            Vec<VEC> xv[U];
            float ck[U];
#pragma unroll
            for (int k = 0; k < U; ++k) {
                const int jj = j + k;
                const int u = __shfl_sync(FULL, u_l, jj & 31);
                if constexpr (COEF != COEF_NONE || OP == OP_GAT)
                    ck[k] = __shfl_sync(FULL, c_l, jj & 31);
                if (jj < n && active) {
                    xv[k] = ld_vec<VEC>(Xc + (int64_t)u * a.ldx);
                } else {
#pragma unroll
                    for (int c = 0; c < VEC; ++c) xv[k].v[c] = 0.f;
                }
            }
#pragma unroll
            for (int k = 0; k < U; ++k) {
                if (j + k < n) {
#pragma unroll
                    for (int c = 0; c < VEC; ++c) {
                        if constexpr (COEF != COEF_NONE || OP == OP_GAT)
                            acc.v[c] = fmaf(ck[k], xv[k].v[c], acc.v[c]);
                        else
                            acc.v[c] += xv[k].v[c];
                    }
                }
            }
        }
    }
}

// Epilogue (a9) for a full row reduction.
template <int VEC, int OP>
__device__ __forceinline__ Vec<VEC> epilogue(const AggArgs &a, int64_t r, int64_t deg, int col,
                                             bool active, const Vec<VEC> &acc, float den) {
    Vec<VEC> y;
    if constexpr (OP == OP_GCN) {
        float cin = 1.f;
        const float dc = (float)(deg > 1 ? deg : 1);
        if (a.norm == TLP_NORM_RIGHT) cin = 1.0f / dc;
        else if (a.norm == TLP_NORM_BOTH) cin = 1.0f / sqrtf(dc);
#pragma unroll
        for (int c = 0; c < VEC; ++c) y.v[c] = acc.v[c] * cin;
    } else if constexpr (OP == OP_GIN) {
        Vec<VEC> xs;
        if (active) xs = ld_vec<VEC>(a.X + (a.row_offset + r) * a.ldx + col);
        else {
#pragma unroll
            for (int c = 0; c < VEC; ++c) xs.v[c] = 0.f;
        }
#pragma unroll
        for (int c = 0; c < VEC; ++c) y.v[c] = fmaf(a.eps1, xs.v[c], acc.v[c]);
    } else {
#pragma unroll
        for (int c = 0; c < VEC; ++c) y.v[c] = deg > 0 ? acc.v[c] / den : 0.f;
    }
    return y;
}

// A regular work unit: whole rows [r0, r1).
template <int VEC, int OP, int COEF, int U>
__device__ __forceinline__ void do_unit(const AggArgs &a, int r0, int r1, int lane) {
    for (int rb = r0; rb < r1; rb += 31) {
        const int nr = min(31, r1 - rb);
        // lanes fetch the row offsets of up to 31 rows at once (register caching
        // of the index boundary, Fig. 7a)
        int64_t rp = 0;
        if (lane <= nr) rp = __ldg(a.rowptr + rb + lane);
        float erl = 0.f;
        if constexpr (OP == OP_GAT)
            if (lane < nr) erl = __ldg(a.er + a.row_offset + rb + lane);
        for (int k = 0; k < nr; ++k) {
            const int64_t e0 = __shfl_sync(FULL, rp, k);
            const int64_t e1 = __shfl_sync(FULL, rp, k + 1);
            const float er_v = (OP == OP_GAT) ? __shfl_sync(FULL, erl, k) : 0.f;
            const int64_t r = rb + k;
            float *yrow = a.Y + r * a.ldy;
            for (int s = 0; s < a.n_strips; ++s) {
                const int col = s * 32 * VEC + lane * VEC;
                const bool active = col < a.F;
                Vec<VEC> acc;
#pragma unroll
                for (int c = 0; c < VEC; ++c) acc.v[c] = 0.f;
                float m = -INFINITY, den = 0.f;
                reduce_edges<VEC, OP, COEF, U>(a, e0, e1, col, active, er_v, lane, acc, m, den);
                Vec<VEC> y = epilogue<VEC, OP>(a, r, e1 - e0, col, active, acc, den);
                if (active) st_row<VEC>(yrow, col, a.F, y);
            }
        }
    }
}

// One C-edge chunk of hub h (a8).  The last chunk to finish merges all the
// partials of the hub in chunk order and writes the row.
template <int VEC, int OP, int COEF, int U>
__device__ __forceinline__ void do_hub_chunk(const AggArgs &a, int h, int j, int lane) {
    const int r = __ldg(a.hub_row + h);
    const int off = __ldg(a.hub_off + h);
    const int nch = __ldg(a.hub_off + h + 1) - off;
    const int64_t eb = __ldg(a.rowptr + r), ee = __ldg(a.rowptr + r + 1);
    const int64_t e0 = eb + (int64_t)j * a.C;
    const int64_t e1 = min(e0 + a.C, ee);
    float er_v = 0.f;
    if constexpr (OP == OP_GAT) er_v = __ldg(a.er + a.row_offset + r);
    const int slot = off + j;
    for (int s = 0; s < a.n_strips; ++s) {
        const int col = s * 32 * VEC + lane * VEC;
        const bool active = col < a.F;
        Vec<VEC> acc;
#pragma unroll
        for (int c = 0; c < VEC; ++c) acc.v[c] = 0.f;
        float m = -INFINITY, den = 0.f;
        reduce_edges<VEC, OP, COEF, U>(a, e0, e1, col, active, er_v, lane, acc, m, den);
        if (active) st_vec<VEC>(a.scratch + (int64_t)slot * a.ldp + col, acc);
        if constexpr (OP == OP_GAT)
            if (s == 0 && lane == 0) {
                a.md[2 * (int64_t)slot] = m;
                a.md[2 * (int64_t)slot + 1] = den;
            }
    }
    __threadfence();
    __syncwarp();
    int last = 0;
    if (lane == 0) last = (atomicAdd(a.hub_ticket + h, 1) == nch - 1);
    last = __shfl_sync(FULL, last, 0);
    if (!last) return;
    __threadfence();
    float *yrow = a.Y + (int64_t)r * a.ldy;
    float M = -INFINITY, D = 0.f;
    if constexpr (OP == OP_GAT) {
        for (int q = 0; q < nch; ++q) M = fmaxf(M, __ldcg(a.md + 2 * (int64_t)(off + q)));
        for (int q = 0; q < nch; ++q) {
            const float mq = __ldcg(a.md + 2 * (int64_t)(off + q));
            const float dq = __ldcg(a.md + 2 * (int64_t)(off + q) + 1);
            D = fmaf(dq, __expf(mq - M), D);
        }
    }
    for (int s = 0; s < a.n_strips; ++s) {
        const int col = s * 32 * VEC + lane * VEC;
        const bool active = col < a.F;
        Vec<VEC> acc;
#pragma unroll
        for (int c = 0; c < VEC; ++c) acc.v[c] = 0.f;
        if (active) {
            for (int q = 0; q < nch; ++q) {
                Vec<VEC> p = ld_vec_cg<VEC>(a.scratch + (int64_t)(off + q) * a.ldp + col);
                if constexpr (OP == OP_GAT) {
                    const float w = __expf(__ldcg(a.md + 2 * (int64_t)(off + q)) - M);
#pragma unroll
                    for (int c = 0; c < VEC; ++c) acc.v[c] = fmaf(w, p.v[c], acc.v[c]);
                } else {
#pragma unroll
                    for (int c = 0; c < VEC; ++c) acc.v[c] += p.v[c];
                }
            }
        }
        Vec<VEC> y = epilogue<VEC, OP>(a, r, ee - eb, col, active, acc, D);
        if (active) st_row<VEC>(yrow, col, a.F, y);
    }
    if (lane == 0) a.hub_ticket[h] = 0;  // self-reset for the next launch
}

template <int VEC, int OP, int COEF, int U>
__device__ __forceinline__ void do_task(const AggArgs &a, int64_t t, int lane) {
    const int2 tk = a.tasks[t];
    if (tk.y >= 0) do_unit<VEC, OP, COEF, U>(a, tk.x, tk.y, lane);
    else do_hub_chunk<VEC, OP, COEF, U>(a, tk.x, -tk.y - 1, lane);
}

template <int VEC, int OP, int COEF, int U>
__global__ void __launch_bounds__(512, 1) k_agg(const AggArgs a) {
    const int lane = threadIdx.x & 31;
    const int64_t wid = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
    if (a.sched == S_HARDWARE) {  // one warp per task
        if (wid < a.n_tasks) do_task<VEC, OP, COEF, U>(a, wid, lane);
        return;
    }
    const int64_t W = ((int64_t)gridDim.x * blockDim.x) >> 5;
    const int64_t stride = W * a.step;
    int64_t t = wid * a.step;  // static first wave
    while (t < a.n_tasks) {
        unsigned long long v = 0;
        if (a.sched == S_DYNAMIC && lane == 0) v = atomicAdd(a.ctr, (unsigned long long)a.step);
        const int64_t tend = min(t + a.step, a.n_tasks);
        for (int64_t tt = t; tt < tend; ++tt) do_task<VEC, OP, COEF, U>(a, tt, lane);
        if (a.sched == S_DYNAMIC) t = stride + (int64_t)__shfl_sync(FULL, v, 0);
        else t += stride;
    }
    if (a.sched == S_DYNAMIC && lane == 0) {
        // last warp out resets the counter: no memset launch between calls
        __threadfence();
        if (atomicAdd(a.done, 1u) == (unsigned)(W - 1)) {
            *a.ctr = 0ull;
            *a.done = 0u;
            __threadfence();
        }
    }
}

// ------------------------------------------------------------- dispatch --

constexpr int kU = 8;  // source rows in flight per warp

typedef void (*KernelFn)(const AggArgs);

template <int VEC>
static KernelFn pick(int op, int coef) {
    if (op == OP_GCN) {
        switch (coef) {
            case COEF_NONE: return k_agg<VEC, OP_GCN, COEF_NONE, kU>;
            case COEF_COUT: return k_agg<VEC, OP_GCN, COEF_COUT, kU>;
            case COEF_W: return k_agg<VEC, OP_GCN, COEF_W, kU>;
            default: return k_agg<VEC, OP_GCN, COEF_W_COUT, kU>;
        }
    }
    if (op == OP_GIN)
        return coef & COEF_W ? k_agg<VEC, OP_GIN, COEF_W, kU> : k_agg<VEC, OP_GIN, COEF_NONE, kU>;
    return k_agg<VEC, OP_GAT, COEF_NONE, kU>;
}

static int occupancy_blocks(KernelFn fn, int threads) {
    // small cache keyed by (kernel, threads)
    struct Entry { KernelFn fn; int threads; int blocks; };
    static thread_local Entry cache[64];
    static thread_local int n_cache = 0;
    for (int i = 0; i < n_cache; ++i)
        if (cache[i].fn == fn && cache[i].threads == threads) return cache[i].blocks;
    int nb = 0;
    if (cudaOccupancyMaxActiveBlocksPerMultiprocessor(&nb, fn, threads, 0) != cudaSuccess || nb < 1)
        nb = 1;
    if (n_cache < 64) cache[n_cache++] = {fn, threads, nb};
    return nb;
}

static bool aligned(const void *p, size_t a) { return ((uintptr_t)p % a) == 0; }

tlp_status aggregate(tlp_graph g, const AggRequest &r, cudaStream_t s) {
    if (!g) return set_error(TLP_ERR_INVALID_ARGUMENT, "null graph");
    if (r.F < 0) return set_error(TLP_ERR_INVALID_ARGUMENT, "F < 0");
    if (r.F == 0 || g->n_dst == 0) return TLP_OK;
    if (r.F >= (int64_t(1) << 30)) return set_error(TLP_ERR_INVALID_ARGUMENT, "F too large");
    if (!r.X || !r.Y) return set_error(TLP_ERR_INVALID_ARGUMENT, "X or Y is NULL");
    if (r.ldx < r.F || r.ldy < r.F)
        return set_error(TLP_ERR_INVALID_ARGUMENT, "leading dimension smaller than F");
    if (!aligned(r.X, 4) || !aligned(r.Y, 4))
        return set_error(TLP_ERR_INVALID_ARGUMENT, "X and Y must be 4-byte aligned");
    if (r.op == OP_GCN && (r.norm < TLP_NORM_NONE || r.norm > TLP_NORM_BOTH))
        return set_error(TLP_ERR_INVALID_ARGUMENT, "unknown norm");
    if (r.op == OP_GIN && g->row_offset + g->n_dst > g->n_src)
        return set_error(TLP_ERR_INVALID_ARGUMENT, "GIN needs row_offset + n_dst <= n_src");
    if (r.op == OP_GAT && (!r.el || !r.er))
        return set_error(TLP_ERR_INVALID_ARGUMENT, "GAT needs el and er");
    {
        const char *x0 = (const char *)r.X;
        const char *x1 = x0 + sizeof(float) * ((g->n_src ? g->n_src - 1 : 0) * r.ldx + r.F);
        const char *y0 = (const char *)r.Y;
        const char *y1 = y0 + sizeof(float) * ((g->n_dst - 1) * r.ldy + r.F);
        if (g->n_src > 0 && x0 < y1 && y0 < x1)
            return set_error(TLP_ERR_INVALID_ARGUMENT, "X and Y overlap (in-place is unsupported)");
    }
    // vector width from the alignment of both operands (R13)
    int vec = 1;
    if (r.ldx % 4 == 0 && r.ldy % 4 == 0 && aligned(r.X, 16) && aligned(r.Y, 16)) vec = 4;
    else if (r.ldx % 2 == 0 && r.ldy % 2 == 0 && aligned(r.X, 8) && aligned(r.Y, 8)) vec = 2;

    int coef = COEF_NONE;
    if (r.op == OP_GCN && r.norm == TLP_NORM_BOTH) coef |= COEF_COUT;
    if (r.op != OP_GAT && g->ew) coef |= COEF_W;

    AggArgs a;
    a.rowptr = g->rowptr;
    a.colidx = g->colidx;
    a.ew = g->ew;
    a.c_out = g->c_out;
    a.X = r.X;
    a.Y = r.Y;
    a.el = r.el;
    a.er = r.er;
    a.tasks = g->tasks;
    a.hub_row = g->hub_row;
    a.hub_off = g->hub_off;
    a.hub_ticket = g->hub_ticket;
    a.ctr = reinterpret_cast<unsigned long long *>(g->ctr);
    a.done = g->ctr + 2;
    a.ldx = r.ldx;
    a.ldy = r.ldy;
    a.ldp = (r.F + 3) / 4 * 4;
    a.row_offset = g->row_offset;
    a.n_tasks = g->n_tasks;
    a.C = g->C;
    a.F = (int)r.F;
    a.n_strips = (int)((r.F + 32 * vec - 1) / (32 * vec));
    a.norm = r.norm;
    a.eps1 = 1.0f + r.eps;
    a.slope = r.slope;
    a.scratch = nullptr;
    a.md = nullptr;
    if (g->n_chunks > 0) {
        size_t need = sizeof(float) * (size_t)g->n_chunks * (a.ldp + 2) + 64;
        tlp_status st = ensure_scratch(g, need, s);
        if (st != TLP_OK) return st;
        a.scratch = g->scratch;
        a.md = g->scratch + (size_t)g->n_chunks * a.ldp;
    }
    // scheduler
    int sched = g->sched;
    if (sched == TLP_SCHED_PAPER) {
        // software mode when n_vertex > 1M or average degree > 50
        bool sw = g->n_dst > 1000000 || (g->n_dst > 0 && g->nnz > 50 * g->n_dst);
        sched = sw ? S_DYNAMIC : S_HARDWARE;
    }
    int step = g->step;
    if (step <= 0) {
        // Alg. 1's step: enough tasks per atomic for ~32 KB of gathered rows
        double edges_per_task = g->n_tasks ? (double)g->nnz / (double)g->n_tasks : 1.0;
        double bytes = edges_per_task * 4.0 * (double)r.F;
        step = (int)std::min(32.0, std::max(1.0, std::ceil(32768.0 / std::max(bytes, 1.0))));
    }
    a.step = step;
    a.sched = sched;

    KernelFn fn = vec == 4 ? pick<4>(r.op, coef) : vec == 2 ? pick<2>(r.op, coef) : pick<1>(r.op, coef);
    const int wpc = g->warps_per_cta > 0 ? std::min(g->warps_per_cta, 16) : 8;
    const int threads = 32 * wpc;
    int64_t blocks;
    if (sched == S_HARDWARE) {
        blocks = (g->n_tasks + wpc - 1) / wpc;
    } else {
        blocks = (int64_t)occupancy_blocks(fn, threads) * g->num_sms;
        int64_t need = (g->n_tasks + (int64_t)wpc * step - 1) / ((int64_t)wpc * step);
        if (blocks > need) blocks = need;  // tiny graphs: do not launch idle warps
    }
    if (blocks < 1) blocks = 1;
    if (blocks > 0x7fffffff) return set_error(TLP_ERR_UNSUPPORTED, "grid too large");
    fn<<<(unsigned)blocks, threads, 0, s>>>(a);
    cudaError_t e = cudaGetLastError();
    if (e != cudaSuccess) return cuda_error(e, "k_agg launch");
    g->last_stream = s;
    return TLP_OK;
}

}  // namespace tlp

using namespace tlp;

extern "C" {

tlp_status tlp_gcn_aggregate(tlp_graph g, const float *X, int64_t F, int64_t ldx, int norm,
                             float *Y, int64_t ldy, void *stream) {
    AggRequest r;
    r.op = OP_GCN;
    r.X = X; r.F = F; r.ldx = ldx; r.Y = Y; r.ldy = ldy; r.norm = norm;
    return aggregate(g, r, (cudaStream_t)stream);
}

tlp_status tlp_gin_aggregate(tlp_graph g, const float *X, int64_t F, int64_t ldx, float eps,
                             float *Y, int64_t ldy, void *stream) {
    AggRequest r;
    r.op = OP_GIN;
    r.X = X; r.F = F; r.ldx = ldx; r.Y = Y; r.ldy = ldy; r.eps = eps;
    return aggregate(g, r, (cudaStream_t)stream);
}

tlp_status tlp_gat_aggregate(tlp_graph g, const float *X, int64_t F, int64_t ldx, const float *el,
                             const float *er, float slope, float *Y, int64_t ldy, void *stream) {
    AggRequest r;
    r.op = OP_GAT;
    r.X = X; r.F = F; r.ldx = ldx; r.Y = Y; r.ldy = ldy;
    r.el = el; r.er = er; r.slope = slope;
    return aggregate(g, r, (cudaStream_t)stream);
}

}  // extern "C"

// tlp_agg.cu -- aggregation dispatch, the scalar passes around the gather
// kernels (repack / pre-scale, GAT edge softmax, GAT backward passes, hot
// tags, projection sums) and the C ABI of the aggregations.  The gather kernel
// templates live in tlp_agg_kernels.cuh (see its header comment for the
// mapping of TLPGNN's two-level parallelism onto sm_100a).
#include <algorithm>
#include <cstdlib>
#include <cstring>
#include <unistd.h>

#include "tlp_agg_kernels.cuh"

namespace tlp {

// Tuning / measurement knobs (TLP_* environment variables) are read
// from a snapshot taken once per aggregate() call: one pass over the
// environment instead of a getenv scan per knob (host cost of a small call).
struct KnobSnapshot {
    int n = 0;
    const char *kv[32];
};
static thread_local KnobSnapshot g_knobs;
static void snapshot_knobs() {
    g_knobs.n = 0;
    for (char **e = environ; e && *e && g_knobs.n < 32; ++e)
        if ((*e)[0] == 'T' && (*e)[1] == 'L' && (*e)[2] == 'P' && (*e)[3] == '_') g_knobs.kv[g_knobs.n++] = *e;
}
static const char *knob(const char *name) {
    const size_t L = strlen(name);
    for (int i = 0; i < g_knobs.n; ++i)
        if (!strncmp(g_knobs.kv[i], name, L) && g_knobs.kv[i][L] == '=') return g_knobs.kv[i] + L + 1;
    return nullptr;
}

// ------------------------------------------------------------- dispatch --

// gather path: 0 register (full warp), 1 cp.async ring, 2 register with G
// lane groups (G = 2: PAIR half-warps; 4, 8: narrow rows; VEC = 4)
static KernelFn pick_kernel(int path, int vec, int op, int coef, int groups) {
    if (path == 2) {
        if (groups == 8) return pick_g8(op, coef);
        if (groups == 4) return pick_g4(op, coef);
        return pick_g2(op, coef);
    }
    if (path == 1) return vec == 4 ? pick_async_v4(op, coef) : pick_async_v21(vec, op, coef);
    return vec == 4 ? pick_reg_v4(op, coef) : pick_reg_v21(vec, op, coef);
}

static int occupancy_blocks(KernelFn fn, int threads, size_t smem) {
    // small cache keyed by (kernel, threads, smem)
    struct Entry { KernelFn fn; int threads; size_t smem; int blocks; };
    static thread_local Entry cache[64];
    static thread_local int n_cache = 0;
    for (int i = 0; i < n_cache; ++i)
        if (cache[i].fn == fn && cache[i].threads == threads && cache[i].smem == smem)
            return cache[i].blocks;
    if (smem > 0) {
        // opt in to the device maximum once per kernel (never lowered afterwards):
        // the opt-in limit covers static + dynamic shared memory
        int dev = 0, mx = 0;
        cudaGetDevice(&dev);
        cudaDeviceGetAttribute(&mx, cudaDevAttrMaxSharedMemoryPerBlockOptin, dev);
        cudaFuncAttributes fa;
        if (cudaFuncGetAttributes(&fa, fn) == cudaSuccess) mx -= (int)fa.sharedSizeBytes;
        if (cudaFuncSetAttribute(fn, cudaFuncAttributeMaxDynamicSharedMemorySize, mx) != cudaSuccess ||
            cudaFuncSetAttribute(fn, cudaFuncAttributePreferredSharedMemoryCarveout, 100) != cudaSuccess)
            cudaGetLastError();  // the launch reports it if the request does not fit
    }
    int nb = 0;
    if (cudaOccupancyMaxActiveBlocksPerMultiprocessor(&nb, fn, threads, smem) != cudaSuccess || nb < 1)
        nb = 1;
    if (n_cache < 64) cache[n_cache++] = {fn, threads, smem, nb};
    return nb;
}

static bool aligned(const void *p, size_t a) { return ((uintptr_t)p % a) == 0; }

// Gather copy of X: out[u, f] = c_out[u] * X[u, f]
// (unweighted GCN BOTH pre-scaling; c_out = NULL copies) for f < F, written
// row-major with leading dimension out_ld, or (pw > 0) panel-major: column f
// of row u at out + (f / pw) * gps + u * pw + f % pw.  The pad columns of the
// last vector are zeroed (they are gathered, never stored to Y).
template <int VEC>
__global__ void k_repack(const float *__restrict__ X, const float *__restrict__ c_out, int64_t n,
                         int64_t F, int64_t ldx, int64_t nvec, float *__restrict__ out,
                         int64_t out_ld, int pw, int64_t gps) {
    const int64_t tot = n * nvec;
    for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < tot;
         i += (int64_t)gridDim.x * blockDim.x) {
        const int64_t u = i / nvec;
        const int64_t c = (i - u * nvec) * VEC;
        const float cu = c_out ? __ldg(c_out + u) : 1.0f;
        const float *src = X + u * ldx + c;
        float *dst = pw ? out + (c / pw) * gps + u * pw + (c % pw) : out + u * out_ld + c;
        if constexpr (VEC == 4) {
            if (c + 4 <= F) {
                const float4 x = __ldg(reinterpret_cast<const float4 *>(src));
                *reinterpret_cast<float4 *>(dst) = make_float4(cu * x.x, cu * x.y, cu * x.z, cu * x.w);
                continue;
            }
        } else if constexpr (VEC == 2) {
            if (c + 2 <= F) {
                const float2 x = __ldg(reinterpret_cast<const float2 *>(src));
                *reinterpret_cast<float2 *>(dst) = make_float2(cu * x.x, cu * x.y);
                continue;
            }
        }
        for (int k = 0; k < VEC; ++k) dst[k] = (c + k < F) ? cu * __ldg(src + k) : 0.f;
    }
}

// NEXT-3: el_out[v] / er_out[v] = sum over strips (in strip order) of the
// epilogue's partial dots.
__global__ void k_proj_sum(const float *__restrict__ proj, int n_strips, int64_t n_dst,
                           float *__restrict__ el_out, float *__restrict__ er_out) {
    for (int64_t v = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; v < n_dst;
         v += (int64_t)gridDim.x * blockDim.x) {
        float l = 0.f, rr = 0.f;
        for (int k = 0; k < n_strips; ++k) {
            const float2 p = *reinterpret_cast<const float2 *>(proj + ((int64_t)k * n_dst + v) * 2);
            l += p.x;
            rr += p.y;
        }
        if (el_out) el_out[v] = l;
        if (er_out) er_out[v] = rr;
    }
}

// GAT edge-softmax pre-pass: per
// local row v, over its in-edges, s_e = LeakyReLU(el[u_e] + er[v]),
// m_v = max_e s_e, z_v = sum_e exp(s_e - m_v), then alpha_e = exp(s_e - m_v) /
// z_v written in CSR edge order (the oracle's two-pass softmax).
// The aggregation then streams alpha as an edge weight.
//   blocks [0, n_hubs): one hub row (in-degree > H) per CTA, thread-strided
//     edges, fixed-order block reduction (a 20K-edge hub does not serialise
//     one warp);
//   blocks [n_hubs, grid): warp per regular row.
// Pass 1 gathers 8 scores per thread per step (8 independent colidx -> el
// chains in flight) and parks s_e in alpha[e]; pass 2 re-reads them (the same
// thread's own stores, L2-resident: no dependent gather) and writes alpha_e.
// Deterministic; hub-ness depends only on the degree and H, so a row slice
// (dist) produces the same bits.
constexpr int kAlphaUnroll = 8;

template <int NT>
__device__ __forceinline__ void alpha_row(const int32_t *__restrict__ colidx, const float *__restrict__ el,
                                          int64_t e0, int64_t e1, float er_v, float slope, int tid,
                                          float *alpha, float *red) {
    constexpr int UN = kAlphaUnroll;
    const int lane = tid & 31;
    float m = -INFINITY, z = 0.f;
    for (int64_t b = e0 + tid; b < e1; b += (int64_t)NT * UN) {
        int c[UN];
#pragma unroll
        for (int k = 0; k < UN; ++k) c[k] = (b + k * NT < e1) ? __ldg(colidx + b + k * NT) : -1;
        float sc[UN];
        float mk = -INFINITY;
#pragma unroll
        for (int k = 0; k < UN; ++k) {
            sc[k] = -INFINITY;
            if (c[k] >= 0) {
                const float t = __ldg(el + c[k]) + er_v;
                sc[k] = t >= 0.f ? t : slope * t;  // LeakyReLU (R6)
                alpha[b + k * NT] = sc[k];
            }
            mk = fmaxf(mk, sc[k]);
        }
        if (mk > m) {  // one rescale per step
            z *= __expf(m - mk);
            m = mk;
        }
#pragma unroll
        for (int k = 0; k < UN; ++k) z += __expf(sc[k] - m);  // exp(-inf) = 0
    }
    float M = warp_max(m);
    float Z = warp_sum(m == -INFINITY ? 0.f : z * __expf(m - M));
    if constexpr (NT > 32) {
        const int w = tid >> 5;
        if (lane == 0) { red[w] = M; red[8 + w] = Z; }
        __syncthreads();
        const float mw = lane < NT / 32 ? red[lane] : -INFINITY;
        const float zw = lane < NT / 32 ? red[8 + lane] : 0.f;
        M = warp_max(mw);
        Z = warp_sum(mw == -INFINITY ? 0.f : zw * __expf(mw - M));
    }
    const float iz = 1.0f / Z;  // unused when the row has no edges
    for (int64_t b = e0 + tid; b < e1; b += (int64_t)NT * UN) {
        float sc[UN];
#pragma unroll
        for (int k = 0; k < UN; ++k)
            if (b + k * NT < e1) sc[k] = alpha[b + k * NT];
#pragma unroll
        for (int k = 0; k < UN; ++k)
            if (b + k * NT < e1) __stcg(alpha + b + k * NT, __expf(sc[k] - M) * iz);
    }
}

__global__ void __launch_bounds__(256) k_gat_alpha(const int64_t *__restrict__ rowptr,
                                                   const int32_t *__restrict__ colidx, int64_t n_dst,
                                                   const float *__restrict__ el, const float *__restrict__ er,
                                                   float slope, const int32_t *__restrict__ hub_row,
                                                   int64_t n_hubs, int64_t H, float *alpha) {
    __shared__ float red[16];
    if ((int64_t)blockIdx.x < n_hubs) {
        const int r = __ldg(hub_row + blockIdx.x);
        alpha_row<256>(colidx, el, __ldg(rowptr + r), __ldg(rowptr + r + 1), __ldg(er + r), slope,
                       threadIdx.x, alpha, red);
        return;
    }
    const int lane = threadIdx.x & 31;
    const int64_t W = ((int64_t)(gridDim.x - n_hubs) * blockDim.x) >> 5;
    for (int64_t v = (((int64_t)blockIdx.x - n_hubs) * blockDim.x + threadIdx.x) >> 5; v < n_dst; v += W) {
        const int64_t e0 = __ldg(rowptr + v), e1 = __ldg(rowptr + v + 1);
        if (e1 - e0 > H) continue;  // a hub: its own CTA
        alpha_row<32>(colidx, el, e0, e1, __ldg(er + v), slope, lane, alpha, red);
    }
}

// ---- GAT backward (NEXT-4) scalar passes -------------------------------------
// The passes around the OP_GATB aggregation:
//  k_gatb_stats (forward rows v): softmax state m_v, z_v of the forward scores
//    and S_v = <dY[v], Y[v]> = sum_e alpha_e g_e, packed with er[v];
//  k_gatb_alpha (transposed rows u): alpha_e, stored in transposed edge order;
//  OP_GATB k_agg (transposed rows u): dX[u] = sum_e alpha_e dY[v_e] and the
//    per-strip dots g_e = dY[v_e] . X[u], one gather of dY per edge;
//  k_gatb_edges (transposed rows u): dt_e = alpha_e (g_e - S_v) LeakyReLU'(t_e),
//    del[u] = sum_e dt_e;  k_gatb_der (forward rows v): der[v] = sum_e dt_e.
// Row-parallel scalar passes: hub rows (degree > H of the handle whose CSR is
// walked) get one 256-thread CTA each (blocks [0, n_hubs)), the other rows a
// warp each; edges are lane-strided with GB_UN independent loads in flight per
// thread.  Sums use a fixed tree (warp butterfly, then warps in order), so
// every pass is deterministic.
constexpr int GB_UN = 4;

template <int NT>
__device__ __forceinline__ float group_sum(float v, float *red, int tid) {
    v = warp_sum(v);
    if constexpr (NT > 32) {
        __syncthreads();  // red is reused by consecutive reductions
        if ((tid & 31) == 0) red[tid >> 5] = v;
        __syncthreads();
        v = ((tid & 31) < NT / 32) ? red[tid & 31] : 0.f;
        v = warp_sum(v);
    }
    return v;
}
template <int NT>
__device__ __forceinline__ void group_max_sum(float &m, float &z, float *red, int tid) {
    float M = warp_max(m);
    float Z = warp_sum(m == -INFINITY ? 0.f : z * __expf(m - M));
    if constexpr (NT > 32) {
        __syncthreads();
        if ((tid & 31) == 0) { red[tid >> 5] = M; red[8 + (tid >> 5)] = Z; }
        __syncthreads();
        const float mw = ((tid & 31) < NT / 32) ? red[tid & 31] : -INFINITY;
        const float zw = ((tid & 31) < NT / 32) ? red[8 + (tid & 31)] : 0.f;
        M = warp_max(mw);
        Z = warp_sum(mw == -INFINITY ? 0.f : zw * __expf(mw - M));
    }
    m = M;
    z = Z;
}

// Dispatch of a row body over the hub CTAs and the warp-per-row blocks.
#define TLP_ROWS(ROWPTR, NROWS, HUBROW, NHUBS, H, BODY)                                         \
    do {                                                                                          \
        __shared__ float red_[16];                                                                \
        if ((int64_t)blockIdx.x < (NHUBS)) {                                                      \
            const int64_t row_ = __ldg((HUBROW) + blockIdx.x);                                    \
            BODY<256>(row_, __ldg((ROWPTR) + row_), __ldg((ROWPTR) + row_ + 1), threadIdx.x, red_); \
            return;                                                                               \
        }                                                                                         \
        const int64_t W_ = ((int64_t)(gridDim.x - (NHUBS)) * blockDim.x) >> 5;                   \
        for (int64_t v_ = (((int64_t)blockIdx.x - (NHUBS)) * blockDim.x + threadIdx.x) >> 5;      \
             v_ < (NROWS); v_ += W_) {                                                            \
            const int64_t a_ = __ldg((ROWPTR) + v_), b_ = __ldg((ROWPTR) + v_ + 1);               \
            if (b_ - a_ > (H)) continue;                                                          \
            BODY<32>(v_, a_, b_, threadIdx.x & 31, red_);                                         \
        }                                                                                         \
    } while (0)

struct GatbStats {
    const int32_t *colidx;
    const float *el, *er, *dY, *Y;
    float slope;
    int64_t lddy, ldy, F;
    float4 *vstat;
    template <int NT>
    __device__ __forceinline__ void operator()(int64_t v, int64_t e0, int64_t e1, int tid, float *red) const {
        const float er_v = __ldg(er + v);
        float m = -INFINITY, z = 0.f;
        for (int64_t b = e0 + tid; b < e1; b += (int64_t)NT * GB_UN) {
            float sc[GB_UN];
            float mk = -INFINITY;
#pragma unroll
            for (int k = 0; k < GB_UN; ++k) {
                sc[k] = -INFINITY;
                if (b + k * NT < e1) {
                    const float t = __ldg(el + __ldg(colidx + b + k * NT)) + er_v;
                    sc[k] = t >= 0.f ? t : slope * t;
                }
                mk = fmaxf(mk, sc[k]);
            }
            if (mk > m) {
                z *= __expf(m - mk);
                m = mk;
            }
#pragma unroll
            for (int k = 0; k < GB_UN; ++k) z += __expf(sc[k] - m);
        }
        group_max_sum<NT>(m, z, red, tid);
        float S = 0.f;
        for (int64_t f = tid; f < F; f += NT) S = fmaf(__ldg(dY + v * lddy + f), __ldg(Y + v * ldy + f), S);
        S = group_sum<NT>(S, red, tid);
        if (tid == 0) vstat[v] = make_float4(er_v, m, z > 0.f ? 1.0f / z : 0.f, S);
    }
};
struct GatbAlpha {
    const int32_t *t_colidx;
    const float *el;
    const float4 *vstat;
    float slope;
    float *alpha;
    template <int NT>
    __device__ __forceinline__ void operator()(int64_t u, int64_t e0, int64_t e1, int tid, float *) const {
        const float el_u = __ldg(el + u);
        for (int64_t b = e0 + tid; b < e1; b += (int64_t)NT * GB_UN) {
            float4 q[GB_UN];
#pragma unroll
            for (int k = 0; k < GB_UN; ++k)
                if (b + k * NT < e1) q[k] = __ldg(vstat + __ldg(t_colidx + b + k * NT));
#pragma unroll
            for (int k = 0; k < GB_UN; ++k)
                if (b + k * NT < e1) {
                    const float t = el_u + q[k].x;
                    const float sc = t >= 0.f ? t : slope * t;
                    alpha[b + k * NT] = __expf(sc - q[k].y) * q[k].z;
                }
        }
    }
};
struct GatbEdges {
    const int32_t *t_colidx;
    const float *el;
    const float4 *vstat;
    const float *alpha;
    float slope;
    const float *gbuf;
    int n_strips;
    int64_t gstride;
    float *dt, *del;
    template <int NT>
    __device__ __forceinline__ void operator()(int64_t u, int64_t e0, int64_t e1, int tid, float *red) const {
        const float el_u = __ldg(el + u);
        float acc = 0.f;
        for (int64_t b = e0 + tid; b < e1; b += (int64_t)NT * GB_UN) {
            float4 q[GB_UN];
            float g[GB_UN], al[GB_UN];
#pragma unroll
            for (int k = 0; k < GB_UN; ++k) {
                g[k] = 0.f;
                if (b + k * NT < e1) {
                    q[k] = __ldg(vstat + __ldg(t_colidx + b + k * NT));
                    al[k] = __ldg(alpha + b + k * NT);
                }
            }
            for (int s = 0; s < n_strips; ++s) {  // strip order (deterministic)
                const float *gs = gbuf + (int64_t)s * gstride;
#pragma unroll
                for (int k = 0; k < GB_UN; ++k)
                    if (b + k * NT < e1) g[k] += __ldcs(gs + b + k * NT);
            }
#pragma unroll
            for (int k = 0; k < GB_UN; ++k)
                if (b + k * NT < e1) {
                    const float t = el_u + q[k].x;
                    const float d = al[k] * (g[k] - q[k].w) * (t >= 0.f ? 1.f : slope);
                    dt[b + k * NT] = d;
                    acc += d;
                }
        }
        acc = group_sum<NT>(acc, red, tid);
        if (tid == 0) del[u] = acc;
    }
};
struct GatbDer {
    const int32_t *tpos;
    const float *dt;
    float *der;
    template <int NT>
    __device__ __forceinline__ void operator()(int64_t v, int64_t e0, int64_t e1, int tid, float *red) const {
        float acc = 0.f;
        for (int64_t b = e0 + tid; b < e1; b += (int64_t)NT * GB_UN * 2) {
            float d[2 * GB_UN];
#pragma unroll
            for (int k = 0; k < 2 * GB_UN; ++k)
                d[k] = (b + k * NT < e1) ? __ldcg(dt + __ldg(tpos + b + k * NT)) : 0.f;
#pragma unroll
            for (int k = 0; k < 2 * GB_UN; ++k) acc += d[k];
        }
        acc = group_sum<NT>(acc, red, tid);
        if (tid == 0) der[v] = acc;
    }
};

#define TLP_BODY(F) F.template operator()
__global__ void __launch_bounds__(256) k_gatb_stats(GatbStats p, const int64_t *__restrict__ rowptr,
                                                    int64_t n, const int32_t *__restrict__ hub_row,
                                                    int64_t n_hubs, int64_t H) {
    TLP_ROWS(rowptr, n, hub_row, n_hubs, H, TLP_BODY(p));
}
__global__ void __launch_bounds__(256) k_gatb_alpha(GatbAlpha p, const int64_t *__restrict__ rowptr,
                                                    int64_t n, const int32_t *__restrict__ hub_row,
                                                    int64_t n_hubs, int64_t H) {
    TLP_ROWS(rowptr, n, hub_row, n_hubs, H, TLP_BODY(p));
}
__global__ void __launch_bounds__(256) k_gatb_edges(GatbEdges p, const int64_t *__restrict__ rowptr,
                                                    int64_t n, const int32_t *__restrict__ hub_row,
                                                    int64_t n_hubs, int64_t H) {
    TLP_ROWS(rowptr, n, hub_row, n_hubs, H, TLP_BODY(p));
}
__global__ void __launch_bounds__(256) k_gatb_der(GatbDer p, const int64_t *__restrict__ rowptr,
                                                  int64_t n, const int32_t *__restrict__ hub_row,
                                                  int64_t n_hubs, int64_t H) {
    TLP_ROWS(rowptr, n, hub_row, n_hubs, H, TLP_BODY(p));
}
#undef TLP_BODY

// ---- hot-source L2 policy ----------------
// Out-degree class of a source: 0 for d <= 1, else min(31, floor(2 log2 d))
// (half-octave classes).  The class only selects an L2 eviction priority.
__device__ __forceinline__ unsigned out_class(int d) {
    if (d <= 1) return 0u;
    return (unsigned)min(31, (int)floorf(2.0f * log2f((float)d)));
}
__global__ void k_tag_colidx(const int32_t *__restrict__ colidx, const int32_t *__restrict__ out_deg,
                             int64_t nnz, int32_t *__restrict__ out) {
    for (int64_t e = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; e < nnz;
         e += (int64_t)gridDim.x * blockDim.x) {
        const int32_t u = colidx[e];
        out[e] = (int32_t)((unsigned)u | (out_class(out_deg[u]) << 27));
    }
}
__global__ void k_class_hist(const int32_t *__restrict__ out_deg, int64_t n,
                             unsigned long long *__restrict__ hist) {
    __shared__ unsigned long long h[32];
    if (threadIdx.x < 32) h[threadIdx.x] = 0;
    __syncthreads();
    for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n;
         i += (int64_t)gridDim.x * blockDim.x)
        atomicAdd(&h[out_class(out_deg[i])], 1ull);
    __syncthreads();
    if (threadIdx.x < 32 && h[threadIdx.x]) atomicAdd(&hist[threadIdx.x], h[threadIdx.x]);
}

// When the gathered rows of X do not fit in L2, the hottest out-degree classes
// whose rows (sector-rounded) fit in kHotFrac of L2 are gathered evict_last and
// the rest evict_first (measured on products GAT: 10.4 -> 9.7 ms).
// TLP_HOT=<fraction> overrides the budget (0 disables).  *thr = (lowest hot
// class) << 27, or 0 when disabled / not applicable.
constexpr double kHotFrac = 0.5;
static tlp_status hot_threshold(tlp_graph g, int64_t ldx, bool panel, cudaStream_t s,
                                unsigned *thr) {
    *thr = 0;
    const char *e = knob("TLP_HOT");
    // by default not in panel mode: there the whole strip of X is meant to stay in L2
    if (!e && panel) return TLP_OK;
    const double frac = e ? atof(e) : kHotFrac;
    if (frac <= 0.0 || g->n_src >= (int64_t(1) << 27) || g->nnz == 0) return TLP_OK;
    const double row = (double)((4 * ldx + 31) / 32 * 32 + 16);
    const double budget = frac * (double)g->l2_bytes;
    if ((double)g->n_src * row <= budget) return TLP_OK;  // all of X fits: nothing to choose
    if (!g->colidx_tag) {
        int32_t *tag = nullptr;
        unsigned long long *hist = nullptr;
        if (cudaMalloc(&tag, sizeof(int32_t) * g->nnz + 16) != cudaSuccess ||
            cudaMalloc(&hist, sizeof(unsigned long long) * 32) != cudaSuccess) {
            cudaFree(tag);
            cudaGetLastError();
            return set_error(TLP_ERR_OUT_OF_MEMORY, "hot tags");
        }
        cudaMemsetAsync(hist, 0, sizeof(unsigned long long) * 32, s);
        k_tag_colidx<<<g->num_sms * 8, 256, 0, s>>>(g->colidx, g->out_deg, g->nnz, tag);
        k_class_hist<<<g->num_sms * 4, 256, 0, s>>>(g->out_deg, g->n_src, hist);
        g->launches += 2;
        unsigned long long h[32];
        cudaMemcpyAsync(h, hist, sizeof(h), cudaMemcpyDeviceToHost, s);
        cudaError_t ce = cudaStreamSynchronize(s);
        cudaFree(hist);
        if (ce != cudaSuccess) {
            cudaFree(tag);
            return cuda_error(ce, "hot tags");
        }
        for (int c = 0; c < 32; ++c) g->tag_hist[c] = (int64_t)h[c];
        g->colidx_tag = tag;
    }
    double used = 0.0;
    int cmin = 32;
    for (int c = 31; c >= 1; --c) {
        const double b = (double)g->tag_hist[c] * row;
        if (used + b > budget) break;
        used += b;
        cmin = c;
    }
    if (cmin < 32) *thr = (unsigned)cmin << 27;
    return TLP_OK;
}

tlp_status aggregate(tlp_graph g, const AggRequest &r, cudaStream_t s) {
    if (!g) return set_error(TLP_ERR_INVALID_ARGUMENT, "null graph");
    snapshot_knobs();
    if (r.F < 0) return set_error(TLP_ERR_INVALID_ARGUMENT, "F < 0");
    if (r.F == 0 || g->n_dst == 0) return TLP_OK;
    if (r.F >= (int64_t(1) << 30)) return set_error(TLP_ERR_INVALID_ARGUMENT, "F too large");
    if (!r.X || !r.Y) return set_error(TLP_ERR_INVALID_ARGUMENT, "X or Y is NULL");
    if (r.ldx < r.F || r.ldy < r.F)
        return set_error(TLP_ERR_INVALID_ARGUMENT, "leading dimension smaller than F");
    if (!aligned(r.X, 4) || !aligned(r.Y, 4))
        return set_error(TLP_ERR_INVALID_ARGUMENT, "X and Y must be 4-byte aligned");
    if (r.op == OP_GCN && (r.norm < TLP_NORM_NONE || r.norm > kNormLeft))
        return set_error(TLP_ERR_INVALID_ARGUMENT, "unknown norm");
    if ((r.op == OP_GIN || (r.op == OP_SAGE && r.sage_self)) && g->row_offset + g->n_dst > g->n_src)
        return set_error(TLP_ERR_INVALID_ARGUMENT, "the self term needs row_offset + n_dst <= n_src");
    if ((r.op == OP_GAT || r.op == OP_GATH) && (!r.el || !r.er))
        return set_error(TLP_ERR_INVALID_ARGUMENT, "GAT needs el and er");
    if (r.act < TLP_ACT_NONE || r.act > TLP_ACT_ELU)
        return set_error(TLP_ERR_INVALID_ARGUMENT, "unknown activation");
    if (r.op < OP_GCN || r.op > OP_GATB)
        return set_error(TLP_ERR_INVALID_ARGUMENT, "unknown op");
    const bool want_proj = r.el_out || r.er_out;
    if ((r.el_out && !r.att_l) || (r.er_out && !r.att_r) || ((r.att_l || r.att_r) && !want_proj))
        return set_error(TLP_ERR_INVALID_ARGUMENT, "epilogue projection needs att_* with *_out");
    if (want_proj && (r.op == OP_GATH || r.op == OP_GATB || r.n_dests > 0))
        return set_error(TLP_ERR_UNSUPPORTED,
                         "epilogue projections: single-head ops, single-GPU output only");
    if (r.op == OP_GATB && (!r.alpha || !r.xself || r.ldxs < r.F || !r.gbuf_out))
        return set_error(TLP_ERR_INVALID_ARGUMENT, "GAT backward arguments");
    if (r.op == OP_GATH && (r.heads < 1 || r.F % r.heads != 0))
        return set_error(TLP_ERR_INVALID_ARGUMENT, "multi-head GAT needs F = heads * head_dim");
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
    {
        // OP_GATB also loads the row's own forward features with the same vectors
        const int64_t lds = (r.op == OP_GATB) ? r.ldxs : 4;
        const void *ps = (r.op == OP_GATB) ? (const void *)r.xself : (const void *)r.X;
        if (r.ldx % 4 == 0 && r.ldy % 4 == 0 && lds % 4 == 0 && aligned(r.X, 16) &&
            aligned(r.Y, 16) && aligned(ps, 16))
            vec = 4;
        else if (r.ldx % 2 == 0 && r.ldy % 2 == 0 && lds % 2 == 0 && aligned(r.X, 8) &&
                 aligned(r.Y, 8) && aligned(ps, 8))
            vec = 2;
    }
    const int fh = (r.op == OP_GATH) ? (int)(r.F / r.heads) : 0;
    if (r.op == OP_GATH)  // a lane's vector may straddle at most two heads
        while (vec > fh) vec >>= 1;

    // Edge coefficients.  GCN BOTH streams the per-edge product
    // c_out[colidx[e]] * w_e precomputed at create (the same fp32 value the
    // kernel would form, so bitwise identical), instead of a dependent gather.
    int coef = COEF_NONE;
    bool prescale = false;
    const float *ew = g->ew;
    const float *cvec = g->c_out;
    int norm = r.norm;
    if (r.op == OP_GCN && r.norm == kNormLeft) {
        // internal: per-source 1/max(d_out,1) gathered per edge, no row scale
        cvec = g->c_out_left;
        coef |= COEF_COUT;
        if (g->ew) coef |= COEF_W;
        norm = TLP_NORM_NONE;
    } else if (r.op == OP_GCN && r.norm == TLP_NORM_BOTH) {
        if (g->ew) {
            ew = g->ew_both;  // weighted: w_e c_out[u] streamed per edge
            coef |= COEF_W;
        } else {
            // unweighted: when the gathered
            // rows are L2-served (X fits, or its 64-column panels do), gather
            // X' = c_out (.) X with no edge coefficient (GIN's register budget);
            // when they stream from HBM, the extra pass over X (read + write of
            // n_src x F) costs more than streaming ew_both[e] = c_out[colidx[e]]
            // (built once per handle).  The choice depends on n_src, ldx and
            // the L2 size only (never on P or the gather path override).
            // TLP_BOTH=prescale|edge overrides.
            // pre-scale only where the L2-panel gathers need a copy of X anyway
            // (DESIGN.md "Gather layout"); when X fits in L2 the extra pass is
            // a launch and a full read + write of X for a latency-bound call
            // (Cora: 37.6 -> 35.5 us without it)
            const double budget = 0.6 * (double)g->l2_bytes;
            bool edge = !(4.0 * (double)g->n_src * (double)r.ldx > budget &&
                          256.0 * (double)g->n_src <= budget);
            if (const char *e = knob("TLP_BOTH")) {
                if (!strcmp(e, "prescale")) edge = false;
                else if (!strcmp(e, "edge")) edge = true;
            }
            if (edge) {
                tlp_status st = ensure_edge_both(g, s);
                if (st != TLP_OK) return st;
                ew = g->ew_both;
                coef |= COEF_W;
            } else {
                prescale = true;
            }
        }
    } else if (r.op != OP_GAT && r.op != OP_GATB && g->ew) {
        coef |= COEF_W;
    }
    if (r.op == OP_GATB) {  // the edge softmax weights, in transposed edge order
        ew = r.alpha;
        coef = COEF_W;
    }
    // GAT edge-softmax pre-pass: when X does not fit in L2 but
    // its 64-column strips do, k_gat_alpha writes every edge's alpha_e once and
    // the aggregation becomes the streamed-weight sum sum_e alpha_e X[u_e] (the
    // GCN-NONE kernel with COEF_W) on the 64-column half-warp panels (the
    // online-softmax kernel would recompute its running state per strip, so it
    // needs 128-column strips that do not stay in L2).  Measured: Reddit 30.0
    // -> 27.7 ms; without panels (products: rows streamed from HBM) the online
    // kernel stays ahead (9.67 vs 9.82 ms).  TLP_GAT=online|alpha overrides.
    int op = r.op;
    bool gat_alpha = false;
    bool join_pending = false;  // the GAT pre-pass ran on g->side: s waits for it before the gather
    if (r.op == OP_GAT) {
        const double budget = 0.6 * (double)g->l2_bytes;
        gat_alpha = vec == 4 && 4.0 * (double)g->n_src * (double)r.ldx > budget &&
                    256.0 * (double)g->n_src <= budget;
        if (const char *e = knob("TLP_GAT")) {
            if (!strcmp(e, "online")) gat_alpha = false;
            else if (!strcmp(e, "alpha")) gat_alpha = true;
        }
        if (gat_alpha && g->nnz > 0) {
            const size_t need = sizeof(float) * (size_t)g->nnz + 64;
            if (need > g->galpha_bytes) {
                if (g->galpha) {
                    cudaFreeAsync(g->galpha, s);
                    g->device_bytes -= g->galpha_bytes;
                    g->galpha = nullptr;
                    g->galpha_bytes = 0;
                }
                cudaError_t e = cudaMallocAsync((void **)&g->galpha, need, s);
                if (e != cudaSuccess) return cuda_error(e, "cudaMallocAsync(GAT alpha)");
                g->galpha_bytes = need;
                g->device_bytes += need;
            }
            const int64_t pb = g->n_hubs + std::max<int64_t>(1, std::min<int64_t>((g->n_dst + 7) / 8, (int64_t)g->num_sms * 16));
            // fork: the pre-pass (latency-bound) overlaps the repack of X
            // (bandwidth-bound) launched next on s; joined before the gather
            // (TLP_GAT_FORK=0: in order on s)
            cudaStream_t sa = s;
            bool fork = true;
            if (const char *e = knob("TLP_GAT_FORK")) fork = atoi(e) != 0;
            if (fork && !g->side) {
                if (cudaStreamCreateWithFlags(&g->side, cudaStreamNonBlocking) != cudaSuccess ||
                    cudaEventCreateWithFlags(&g->ev_fork, cudaEventDisableTiming) != cudaSuccess ||
                    cudaEventCreateWithFlags(&g->ev_join, cudaEventDisableTiming) != cudaSuccess)
                    return cuda_error(cudaGetLastError(), "GAT pre-pass stream");
            }
            if (fork) {
                cudaError_t e = cudaEventRecord(g->ev_fork, s);
                if (e == cudaSuccess) e = cudaStreamWaitEvent(g->side, g->ev_fork, 0);
                if (e != cudaSuccess) return cuda_error(e, "GAT pre-pass fork");
                sa = g->side;
                join_pending = true;
            }
            k_gat_alpha<<<(unsigned)pb, 256, 0, sa>>>(g->rowptr, g->colidx, g->n_dst, r.el, r.er + g->row_offset,
                                                      r.slope, g->hub_row, g->n_hubs, g->H, g->galpha);
            g->launches += 1;
            cudaError_t e = cudaGetLastError();
            if (e != cudaSuccess) return cuda_error(e, "k_gat_alpha launch");
            if (fork) {
                e = cudaEventRecord(g->ev_join, g->side);
                if (e != cudaSuccess) return cuda_error(e, "GAT pre-pass join");
            }
        }
        if (gat_alpha) {
            op = OP_GCN;  // Y[v] = sum_e alpha_e X[u_e]: unnormalised streamed-weight sum
            norm = TLP_NORM_NONE;
            coef = COEF_W;
            ew = g->galpha;
        }
    }
    // Feature panels: when X is much larger than
    // L2, sweep the graph once per column strip so the strip of X being
    // gathered (n_src x strip width x 4 bytes) stays L2-resident while every
    // edge pulls from it.  Strips are 64 columns gathered by half-warps (PAIR:
    // lanes 0-15 and 16-31 take consecutive edges, LDG.128 each) when that
    // slice fits in 60% of L2, else 128 columns (full warp, LDG.128).  The
    // reduction order is the canonical two-chain order in every case, so panel
    // mode and strip width never change a single output bit.
    int panel = 0, pair = 0;  // pair: lane groups of a panel strip (0: none)
    int lps = 32;  // lanes per full-warp strip
    bool panel_off = false;
    {
        const double budget = 0.6 * (double)g->l2_bytes;
        const double xbytes = 4.0 * (double)g->n_src * (double)r.ldx;
        int mode = -1;  // auto
        if (const char *e = knob("TLP_PANEL")) mode = atoi(e);
        if (mode == 0) {
            panel_off = true;
        } else if (mode == 128 && vec == 4) {
            panel = 1;
        } else if (mode == 64 && vec == 4 && r.op != OP_GATH) {
            panel = 1;
            pair = 2;
        } else if (mode == 64 && vec == 2) {
            panel = 1;
        } else if ((mode == 32 || mode == 16) && vec == 4 && r.op != OP_GATH) {
            panel = 1;  // lane-group strips: 32 columns = 4 groups of 8 lanes, 16 = 8 of 4
            pair = 128 / mode;
        } else if (mode == 32) {
            panel = 1;
            vec = 1;
        } else if (mode > 0 && mode < 128 && mode % 4 == 0 && vec == 4 && r.op != OP_GATH) {
            panel = 1;  // narrow full-warp strips of `mode` columns
            lps = mode / 4;
        } else if (xbytes > budget && vec == 4) {
            // online-softmax GAT recomputes its running state per strip, so it
            // keeps the wider 128-column strips (measured)
            if (op != OP_GAT && op != OP_GATH && 256.0 * g->n_src <= budget) {
                panel = 1;
                pair = 2;
            }
            else if (512.0 * g->n_src <= (double)g->l2_bytes) panel = 1;
        }
    }
    // Lane groups: G = 2 for the 64-column PAIR
    // strips; for narrow rows (F/4 vectors fill at most half a warp) G = 2, 4
    // or 8 groups of 32/G lanes each gather their own edge, so every warp
    // instruction still moves up to 512 bytes (F = 32: 4 rows of 128 B).
    // TLP_GROUPS=1|2|4|8 overrides.
    int groups = pair ? pair : 1;
    if (!panel && !pair && lps == 32 && vec == 4 && op != OP_GATH) {
        const int64_t nv = (r.F + 3) / 4;
        groups = nv <= 4 ? 8 : nv <= 8 ? 4 : nv <= 16 ? 2 : 1;
    }
    if (const char *e = knob("TLP_GROUPS")) {
        const int gq = atoi(e);
        if ((gq == 1 || gq == 2 || gq == 4 || gq == 8) && vec == 4 && lps == 32 && op != OP_GATH)
            groups = gq;
    }
    if (op == OP_GATB && groups > 2) groups = 2;  // the edge-dot trees exist for G <= 2
    const int strip_w = groups > 1 ? (32 / groups) * vec : lps * vec;
    const int n_strips = (int)((r.F + strip_w - 1) / strip_w);
    // Few tasks for the resident warps (small graphs): split every task into its
    // strips as separate work items too, so all SMs get work.
    bool spread = false;  // panel set only to spread a small graph's work (not an L2 panel)
    if (!panel && !panel_off && n_strips > 1 && g->n_tasks < (int64_t)g->num_sms * 32 * 4) panel = spread = 1;
    if (n_strips < 2) panel = 0;

    // Gather layout.  In L2-panel mode (X larger
    // than L2, its strips not) every edge gathers one strip of a source row
    // from L2.  A strip that is not 128-byte aligned touches one more cache
    // line and one more sector per gather and inflates the L2 footprint of the
    // panel; a strip spread over all of X (row stride ld) touches every page of
    // X per sweep.  So the gathers read a panel-major copy of X -- strip s is a
    // contiguous [n_src x strip_w] block, 256-byte rows -- written by one
    // streaming pass (read + write of n_src x F, ~1 % of a Reddit launch); the
    // unweighted GCN-BOTH pre-scale writes its X' in that layout at no extra
    // cost.  Measured on Reddit (F = 602): GIN 21.4 ms (caller ld 604) / 17.9
    // (caller ld 608) / 18.4 (padded copy) / 16.7 (panel-major copy), GCN-BOTH
    // 22.3 / 18.8 / 18.8 / 17.2, GAT 24.4 / 20.9 / 21.1 / 19.9.  Values are
    // copied bit for bit (or scaled exactly as before), so no output bit
    // changes.  TLP_LAYOUT=caller|padded|panel overrides (and applies to any
    // panel-mode call, so tests can force it on small inputs).
    int layout = 0;  // 0 caller, 1 padded rows, 2 panel-major
    if (panel && vec == 4 && op != OP_GATH) {
        if (4.0 * (double)g->n_src * (double)r.ldx > 0.6 * (double)g->l2_bytes) layout = 2;
        if (const char *e = knob("TLP_LAYOUT")) {
            if (!strcmp(e, "caller")) layout = 0;
            else if (!strcmp(e, "padded")) layout = 1;
            else if (!strcmp(e, "panel")) layout = 2;
        }
        if (layout == 2 && strip_w % 4 != 0) layout = 1;
    }
    // Unweighted GCN BOTH: one pass writes
    // X'[u] = c_out[u] X[u] (each term rounded once, as the oracle's product),
    // then every gather path sums X' rows with no per-edge coefficient, i.e.
    // the register budget and instruction count of GIN.  Same bits on every
    // path, schedule and partition (every path gathers the same X').
    const float *Xg = r.X;
    int64_t ldg = r.ldx, gps = 0;
    if (prescale || layout != 0) {
        if (layout == 1) ldg = (r.F + 31) / 32 * 32;
        if (layout == 2) {
            ldg = strip_w;
            gps = g->n_src * (int64_t)strip_w;
        }
        const size_t need = sizeof(float) * (layout == 2 ? (size_t)n_strips * (size_t)gps
                                                           : (size_t)g->n_src * (size_t)ldg) + 256;
        if (need > g->xs_bytes) {
            if (g->xs) {
                cudaFreeAsync(g->xs, s);
                g->device_bytes -= g->xs_bytes;
                g->xs = nullptr;
                g->xs_bytes = 0;
            }
            cudaError_t e = cudaMallocAsync((void **)&g->xs, need, s);
            if (e != cudaSuccess) return cuda_error(e, "cudaMallocAsync(prescaled X)");
            g->xs_bytes = need;
            g->device_bytes += need;
        }
        const int64_t nvec = (r.F + vec - 1) / vec;
        const int64_t tot = g->n_src * nvec;
        const int pb = (int)std::max<int64_t>(1, std::min<int64_t>((tot + 255) / 256, (int64_t)g->num_sms * 16));
        const float *cs = prescale ? g->c_out : nullptr;
        const int pw = layout == 2 ? strip_w : 0;
        if (vec == 4)
            k_repack<4><<<pb, 256, 0, s>>>(r.X, cs, g->n_src, r.F, r.ldx, nvec, g->xs, ldg, pw, gps);
        else if (vec == 2)
            k_repack<2><<<pb, 256, 0, s>>>(r.X, cs, g->n_src, r.F, r.ldx, nvec, g->xs, ldg, pw, gps);
        else
            k_repack<1><<<pb, 256, 0, s>>>(r.X, cs, g->n_src, r.F, r.ldx, nvec, g->xs, ldg, pw, gps);
        g->launches += 1;
        cudaError_t e = cudaGetLastError();
        if (e != cudaSuccess) return cuda_error(e, "k_repack launch");
        Xg = g->xs;
    }


    AggArgs a;
    a.rowptr = g->rowptr;
    a.colidx = g->colidx;
    a.ew = ew;
    a.c_out = cvec;
    a.X = Xg;
    a.xown = r.X;
    a.ldown = r.ldx;
    a.gps = gps;
    a.pw = strip_w;
    a.Y = r.Y;
    a.el = r.el;
    a.er = r.er;
    a.tasks = g->tasks;
    a.hub_row = g->hub_row;
    a.hub_off = g->hub_off;
    a.ctr = g->ctr;
    a.done = g->ctr + 2;
    a.ldx = ldg;
    a.ldy = r.ldy;
    a.ldp = (r.F + 3) / 4 * 4;
    a.row_offset = g->row_offset;
    a.n_tasks = g->n_tasks;
    a.tasks_magic = 0;
    a.skip_hubs = 0;
    a.hub_H = g->H;
    a.stream_hint = 0;
    a.visits = g->visits;
    if (g->n_tasks > 1)  // ceil(2^64 / n_tasks)
        a.tasks_magic = (unsigned long long)((((unsigned __int128)1) << 64) / (unsigned __int128)g->n_tasks) + 1ull;
    a.n_hubs = g->n_hubs;
    a.n_chunks = g->n_chunks;
    a.C = g->C;
    a.F = (int)r.F;
    a.n_strips = n_strips;
    a.lps = lps;
    a.panel = panel;
    a.n_items = panel ? g->n_tasks * n_strips : g->n_tasks;
    a.norm = norm;
    a.eps1 = 1.0f + r.eps;
    a.slope = r.slope;
    a.sage_self = r.sage_self;
    a.bias = r.bias;
    a.dests = r.dests;
    a.n_dests = r.n_dests;
    a.mc = r.mc;
    a.hot_thr = 0;
    a.cold_first = 0;
    a.xself = r.xself;
    a.ldxs = r.ldxs;
    a.att_l = r.att_l;
    a.att_r = r.att_r;
    a.proj = nullptr;
    a.n_dst = g->n_dst;
    if (want_proj) {
        const size_t need = sizeof(float) * 2 * (size_t)n_strips * (size_t)g->n_dst + 64;
        if (need > g->proj_bytes) {
            if (g->proj) {
                cudaFreeAsync(g->proj, s);
                g->device_bytes -= g->proj_bytes;
                g->proj = nullptr;
                g->proj_bytes = 0;
            }
            cudaError_t e = cudaMallocAsync((void **)&g->proj, need, s);
            if (e != cudaSuccess) return cuda_error(e, "cudaMallocAsync(projections)");
            g->proj_bytes = need;
            g->device_bytes += need;
        }
        a.proj = g->proj;
    }
    a.gbuf = nullptr;
    a.gstride = g->nnz;
    if (r.op == OP_GATB) {
        const size_t need = sizeof(float) * ((size_t)n_strips * (size_t)g->nnz + 16);
        if (need > g->bwd_bytes) {
            if (g->bwd) {
                cudaFreeAsync(g->bwd, s);
                g->device_bytes -= g->bwd_bytes;
                g->bwd = nullptr;
                g->bwd_bytes = 0;
            }
            cudaError_t e = cudaMallocAsync((void **)&g->bwd, need, s);
            if (e != cudaSuccess) return cuda_error(e, "cudaMallocAsync(gat backward dots)");
            g->bwd_bytes = need;
            g->device_bytes += need;
        }
        a.gbuf = g->bwd;
        *r.gbuf_out = g->bwd;
        if (r.n_strips_out) *r.n_strips_out = n_strips;
    }
    a.act = r.act;
    a.act_param = r.act_param;
    a.heads = (int)r.heads;
    a.fh = fh;
    a.fh_magic = (fh > 1 && r.F < (1 << 16))
                     ? (unsigned)(((uint64_t(1) << 32) + (uint64_t)fh - 1) / (uint64_t)fh)
                     : 0u;
    a.scratch = nullptr;
    a.md = nullptr;
    a.hub_ticket = nullptr;
    if (g->n_chunks > 0) {
        // scratch = [partials n_chunks x ldp][(m,den) 2 x n_chunks x panels][tickets n_hubs x panels]
        const int np = panel ? n_strips : 1;
        const size_t part = (size_t)g->n_chunks * a.ldp;
        const size_t mdn = 2 * (size_t)g->n_chunks * np * (r.op == OP_GATH ? (size_t)r.heads : 1);
        const size_t tick_off = (part + mdn) * sizeof(float);
        const size_t tick_n = (size_t)g->n_hubs * np;
        const size_t need = tick_off + tick_n * sizeof(int32_t) + 64;
        const bool realloc_ = need > g->scratch_bytes;
        tlp_status st = ensure_scratch(g, need, s);
        if (st != TLP_OK) return st;
        if (realloc_ || g->ticket_off != tick_off || g->ticket_n < tick_n) {
            cudaError_t e = cudaMemsetAsync((char *)g->scratch + tick_off, 0,
                                            tick_n * sizeof(int32_t), s);
            if (e != cudaSuccess) return cuda_error(e, "cudaMemsetAsync(tickets)");
            g->ticket_off = tick_off;
            g->ticket_n = tick_n;
        }
        a.scratch = g->scratch;
        a.md = g->scratch + part;
        a.hub_ticket = reinterpret_cast<int32_t *>((char *)g->scratch + tick_off);
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
        // Alg. 1's step: enough work items per atomic for ~32 KB of gathered rows
        double edges_per_task = g->n_tasks ? (double)g->nnz / (double)g->n_tasks : 1.0;
        double width = panel ? (double)strip_w : (double)r.F;
        double bytes = edges_per_task * 4.0 * width;
        step = (int)std::min(32.0, std::max(1.0, std::ceil(32768.0 / std::max(bytes, 1.0))));
        // ... but never so large that the resident warps (~SMs x 24) get fewer
        // than ~4 fetches each: small graphs are latency-bound, spread them out
        const double resident = (double)g->num_sms * 24.0;
        const double cap = std::max(1.0, std::floor((double)a.n_items / (resident * 4.0)));
        step = (int)std::min((double)step, cap);
    }
    a.step = step;
    a.sched = sched;

    // Gather path: gathers served from an
    // L2-resident panel are latency-light and instruction-bound -> register
    // double buffering (full warp, or PAIR half-warps for 64-column strips);
    // gathers that stream from HBM need more bytes in flight than registers can
    // hold -> cp.async shared-memory ring.  TLP_GATHER (reg|async) overrides.
    bool async_path = !panel && (4.0 * (double)g->n_src * (double)r.ldx > 0.6 * (double)g->l2_bytes);
    if (const char *e = knob("TLP_GATHER")) {
        if (!strcmp(e, "reg")) async_path = false;
        else if (!strcmp(e, "async")) async_path = true;
    }
    if (groups > 1 || r.op == OP_GATB) async_path = false;  // OP_GATB: register path only
    const int path = groups > 1 ? 2 : (async_path ? 1 : 0);
    // CLC scheduling is compiled into the register-path kernels only (see
    // agg_clc): the cp.async kernels run it with the atomic counter
    if (sched == S_CLC && async_path) a.sched = sched = S_DYNAMIC;
    // hot-source L2 policy: cp.async path only (rows streamed from HBM)
    if (async_path && r.op != OP_GATB) {
        unsigned thr = 0;
        tlp_status st = hot_threshold(g, panel ? (int64_t)strip_w : r.ldx, panel != 0, s, &thr);
        if (st != TLP_OK) return st;
        if (thr) {
            a.colidx = g->colidx_tag;
            a.hot_thr = thr;
            a.cold_first = 1;
            if (const char *e = knob("TLP_HOT_COLD")) a.cold_first = atoi(e);
        }
    }
    // L2 stream hints in L2-panel mode only;
    // TLP_HINTS=0|1 overrides
    a.stream_hint = (panel && !spread && !async_path) ? 1 : 0;
    if (const char *e = knob("TLP_HINTS")) a.stream_hint = atoi(e) != 0;
    if (join_pending) {
        cudaError_t e = cudaStreamWaitEvent(s, g->ev_join, 0);
        if (e != cudaSuccess) return cuda_error(e, "GAT pre-pass join");
    }
    KernelFn fn = (r.op == OP_GATH) ? pick_mh(vec, async_path) : pick_kernel(path, vec, op, coef, groups);
    const int wpc = g->warps_per_cta > 0 ? std::min(g->warps_per_cta, TLP_MAXT / 32) : 8;
    const int threads = 32 * wpc;
    size_t smem = async_path ? (size_t)wpc * TLP_DEPTH * 32 * vec * sizeof(float) : 0;
    if (r.op == OP_GATH) {
        // heads a 32*vec-column strip can touch: ceil((W - 1) / fh) + 1, at most H
        const int W = 32 * vec;
        a.mh_nh = std::min((int)r.heads, (W - 1 + fh - 1) / fh + 1);
        a.mh_words = (a.mh_nh * 32 + 3 * a.mh_nh + 1 + 3) & ~3;
        smem = (size_t)wpc * (a.mh_words + (async_path ? TLP_DEPTH_MH * 32 * vec : 0)) * sizeof(float);
    }
    // the general persistent kernel over a.n_items work items
    auto launch_general = [&](const AggArgs &ag) -> tlp_status {
        if (smem > 0 && (sched == S_HARDWARE || sched == S_CLC)) occupancy_blocks(fn, threads, smem);  // sets attributes
        int64_t blocks;
        if (sched == S_HARDWARE) {
            blocks = (ag.n_items + wpc - 1) / wpc;
        } else if (sched == S_CLC) {  // one CTA per wpc * step items; running CTAs steal the rest
            blocks = (ag.n_items + (int64_t)wpc * step - 1) / ((int64_t)wpc * step);
        } else {
            int per_sm = occupancy_blocks(fn, threads, smem);
            if (const char *e = knob("TLP_CTAS"))  // measurement: cap resident CTAs per SM
                if (atoi(e) > 0) per_sm = std::min(per_sm, atoi(e));
            blocks = (int64_t)per_sm * g->num_sms;
            int64_t need = (ag.n_items + (int64_t)wpc * step - 1) / ((int64_t)wpc * step);
            if (blocks > need) blocks = need;  // tiny graphs: do not launch idle warps
        }
        if (blocks < 1) blocks = 1;
        if (blocks > 0x7fffffff) return set_error(TLP_ERR_UNSUPPORTED, "grid too large");
        // the kernel walks work items with 32-bit indices
        if (ag.n_items + (blocks * wpc + 1) * (int64_t)std::max(step, 1) >= (int64_t(1) << 31))
            return set_error(TLP_ERR_UNSUPPORTED, "too many work items (tasks x strips >= 2^31)");
        fn<<<(unsigned)blocks, threads, smem, s>>>(ag);
        g->launches += 1;
        cudaError_t e = cudaGetLastError();
        if (e != cudaSuccess) return cuda_error(e, "k_agg launch");
        return TLP_OK;
    };
    // Short-row kernel (tlp_k_rows.cu): one warp per
    // (row, 128-column strip) item, static round-robin, small
    // register footprint, next item's row bounds prefetched.  Used by default
    // for hub-free graphs whose X is L2-resident (latency-bound calls: Cora,
    // Pubmed).  With hub rows the general kernel runs their chunks first and
    // the short-row kernel skips them.  Bitwise the same output as the general
    // kernel (same coefficients, same canonical order), so the choice never
    // changes a result.  TLP_ROWS=0|1 overrides.
    const bool rows_ok = (!panel || spread) && groups == 1 && vec == 4 && lps == 32 &&
                         (op == OP_GCN || op == OP_GIN || op == OP_SAGE || op == OP_GAT) &&
                         r.op != OP_GATH && r.op != OP_GATB;
    bool rows_k = rows_ok && g->n_hubs == 0 && !async_path && !panel_off &&
                  4.0 * (double)g->n_src * (double)r.ldx <= 0.6 * (double)g->l2_bytes &&
                  knob("TLP_PANEL") == nullptr && knob("TLP_GATHER") == nullptr;
    if (const char *e = knob("TLP_ROWS")) rows_k = rows_ok && atoi(e) != 0;
    const int nstr = (int)((r.F + 127) / 128);
    // strips per short-row work item (TLP_ROWS_NSI=1|2 overrides)
    int nsi = nstr >= 2 ? 2 : 1;
    if (const char *e = knob("TLP_ROWS_NSI")) nsi = (atoi(e) == 2) ? 2 : 1;
    // nothing but the aggregation itself: the short-row kernel's lean store path
    const bool plain = a.bias == nullptr && a.act == TLP_ACT_NONE && a.n_dests == 0 && a.mc == nullptr &&
                       a.proj == nullptr && !a.stream_hint && a.visits == nullptr;
    KernelFn fr = rows_k ? pick_rows(op, coef, a.hot_thr != 0, nsi, plain) : nullptr;

    if (fr) {
        const int ipr = (nstr + nsi - 1) / nsi;  // work items per row
        if (g->n_hubs > 0) {  // hub chunks in the general kernel (tasks [0, n_chunks))
            AggArgs ah = a;
            ah.panel = 0;  // task-major: each hub-chunk item covers all strips
            ah.n_items = g->n_chunks;
            tlp_status st = launch_general(ah);
            if (st != TLP_OK) return st;
        }
        AggArgs ar = a;
        // (keeps the hot-source tags and threshold of the cp.async path, if any)
        ar.n_strips = nstr;
        ar.panel = 0;
        ar.skip_hubs = g->n_hubs > 0 ? 1 : 0;
        ar.hub_H = g->H;
        ar.n_items = g->n_dst * (int64_t)ipr;
        ar.tasks_magic = (ipr > 1)
                             ? (unsigned long long)((((unsigned __int128)1) << 64) / (unsigned __int128)ipr) + 1ull
                             : 0ull;
        if (ar.n_items >= (int64_t(1) << 31)) return set_error(TLP_ERR_UNSUPPORTED, "too many rows x strips");
        const int per_sm = occupancy_blocks(fr, 256, 0);
        int64_t nb = std::min<int64_t>((int64_t)per_sm * g->num_sms, (ar.n_items + 7) / 8);
        if (nb < 1) nb = 1;
        fr<<<(unsigned)nb, 256, 0, s>>>(ar);
        g->launches += 1;
        cudaError_t e = cudaGetLastError();
        if (e != cudaSuccess) return cuda_error(e, "k_rows launch");
    } else {
        tlp_status st = launch_general(a);
        if (st != TLP_OK) return st;
    }
    if (want_proj) {
        const int pb = (int)std::min<int64_t>((g->n_dst + 255) / 256, (int64_t)g->num_sms * 8);
        k_proj_sum<<<pb, 256, 0, s>>>(g->proj, n_strips, g->n_dst, r.el_out, r.er_out);
        g->launches += 1;
        cudaError_t e = cudaGetLastError();
        if (e != cudaSuccess) return cuda_error(e, "k_proj_sum launch");
    }
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

// NEXT-4: backward aggregations on the transposed CSR.  dX = M^T dY:
//   GCN BOTH  = GCN BOTH forward of the transpose (its c_out is the forward c_in,
//               its c_in the forward c_out);  NONE = NONE;
//   GCN RIGHT = per-source 1/max(d_out,1) of the transpose (internal LEFT norm);
//   GIN       = GIN forward of the transpose (square graphs).
tlp_status tlp_gcn_backward(tlp_graph g, const float *dY, int64_t F, int64_t lddy, int norm,
                            float *dX, int64_t lddx, void *stream) {
    if (!g) return set_error(TLP_ERR_INVALID_ARGUMENT, "null graph");
    if (!g->t) return set_error(TLP_ERR_INVALID_ARGUMENT, "call tlp_graph_build_transpose first");
    if (norm < TLP_NORM_NONE || norm > TLP_NORM_BOTH)
        return set_error(TLP_ERR_INVALID_ARGUMENT, "unknown norm");
    AggRequest r;
    r.op = OP_GCN;
    r.X = dY; r.F = F; r.ldx = lddy; r.Y = dX; r.ldy = lddx;
    r.norm = (norm == TLP_NORM_RIGHT) ? kNormLeft : norm;
    return aggregate(g->t, r, (cudaStream_t)stream);
}

tlp_status tlp_gin_backward(tlp_graph g, const float *dY, int64_t F, int64_t lddy, float eps,
                            float *dX, int64_t lddx, void *stream) {
    if (!g) return set_error(TLP_ERR_INVALID_ARGUMENT, "null graph");
    if (!g->t) return set_error(TLP_ERR_INVALID_ARGUMENT, "call tlp_graph_build_transpose first");
    if (g->n_src != g->n_dst) return set_error(TLP_ERR_INVALID_ARGUMENT, "GIN backward needs a square graph");
    AggRequest r;
    r.op = OP_GIN;
    r.X = dY; r.F = F; r.ldx = lddy; r.Y = dX; r.ldy = lddx; r.eps = eps;
    return aggregate(g->t, r, (cudaStream_t)stream);
}

tlp_status tlp_gat_backward(tlp_graph g, const float *X, int64_t F, int64_t ldx, const float *el,
                            const float *er, float slope, const float *Y, int64_t ldy,
                            const float *dY, int64_t lddy, float *dX, int64_t lddx, float *del,
                            float *der, void *stream) {
    cudaStream_t s = (cudaStream_t)stream;
    if (!g) return set_error(TLP_ERR_INVALID_ARGUMENT, "null graph");
    if (!g->t) return set_error(TLP_ERR_INVALID_ARGUMENT, "call tlp_graph_build_transpose first");
    if (F < 0) return set_error(TLP_ERR_INVALID_ARGUMENT, "F < 0");
    if (!el || !er || !del || !der || (F > 0 && (!X || !Y || !dY || !dX)))
        return set_error(TLP_ERR_INVALID_ARGUMENT, "NULL argument");
    if (ldx < F || ldy < F || lddy < F || lddx < F)
        return set_error(TLP_ERR_INVALID_ARGUMENT, "leading dimension smaller than F");
    const int64_t n_dst = g->n_dst, n_src = g->n_src, nnz = g->nnz;
    if (F == 0) {  // no features: every gradient is zero
        if (n_src) TLP_CUDA_TRY(cudaMemsetAsync(del, 0, sizeof(float) * n_src, s));
        if (n_dst) TLP_CUDA_TRY(cudaMemsetAsync(der, 0, sizeof(float) * n_dst, s));
        return TLP_OK;
    }
    // forward-graph scratch: vstat [n_dst] float4, then dt [nnz], alpha [nnz]
    const size_t vbytes = ((size_t)n_dst * 16 + 255) / 256 * 256;
    const size_t ebytes = (sizeof(float) * (size_t)nnz + 255) / 256 * 256;
    const size_t need = vbytes + 2 * ebytes + 64;
    if (need > g->bwd_bytes) {
        if (g->bwd) {
            cudaFreeAsync(g->bwd, s);
            g->device_bytes -= g->bwd_bytes;
            g->bwd = nullptr;
            g->bwd_bytes = 0;
        }
        cudaError_t e = cudaMallocAsync((void **)&g->bwd, need, s);
        if (e != cudaSuccess) return cuda_error(e, "cudaMallocAsync(gat backward)");
        g->bwd_bytes = need;
        g->device_bytes += need;
    }
    float4 *vstat = reinterpret_cast<float4 *>(g->bwd);
    float *dt = reinterpret_cast<float *>((char *)g->bwd + vbytes);
    float *alpha = reinterpret_cast<float *>((char *)g->bwd + vbytes + ebytes);
    const int nsm = g->num_sms > 0 ? g->num_sms : 148;
    if (n_dst) {
        GatbStats p{g->colidx, el, er, dY, Y, slope, lddy, ldy, F, vstat};
        k_gatb_stats<<<(unsigned)(g->n_hubs + nsm * 8), 256, 0, s>>>(p, g->rowptr, n_dst, g->hub_row,
                                                                   g->n_hubs, g->H);
        g->launches += 1;
        TLP_CUDA_TRY(cudaGetLastError());
    }
    if (n_src == 0) {
        if (n_dst) TLP_CUDA_TRY(cudaMemsetAsync(der, 0, sizeof(float) * n_dst, s));
        return TLP_OK;
    }
    {
        GatbAlpha p{g->t->colidx, el, vstat, slope, alpha};
        k_gatb_alpha<<<(unsigned)(g->t->n_hubs + nsm * 8), 256, 0, s>>>(p, g->t->rowptr, n_src,
                                                                      g->t->hub_row, g->t->n_hubs, g->t->H);
    }
    g->launches += 1;
    TLP_CUDA_TRY(cudaGetLastError());
    AggRequest r;
    r.op = OP_GATB;
    r.X = dY; r.F = F; r.ldx = lddy; r.Y = dX; r.ldy = lddx;
    r.alpha = alpha;
    r.xself = X; r.ldxs = ldx;
    float *gbuf = nullptr;
    int n_strips = 0;
    r.gbuf_out = &gbuf;
    r.n_strips_out = &n_strips;
    tlp_status st = aggregate(g->t, r, s);
    if (st != TLP_OK) return st;
    {
        GatbEdges p{g->t->colidx, el, vstat, alpha, slope, gbuf, n_strips, nnz, dt, del};
        k_gatb_edges<<<(unsigned)(g->t->n_hubs + nsm * 8), 256, 0, s>>>(p, g->t->rowptr, n_src,
                                                                      g->t->hub_row, g->t->n_hubs, g->t->H);
    }
    g->launches += 1;
    TLP_CUDA_TRY(cudaGetLastError());
    if (n_dst) {
        GatbDer p{g->tpos, dt, der};
        k_gatb_der<<<(unsigned)(g->n_hubs + nsm * 8), 256, 0, s>>>(p, g->rowptr, n_dst, g->hub_row,
                                                                 g->n_hubs, g->H);
        g->launches += 1;
        TLP_CUDA_TRY(cudaGetLastError());
    }
    return TLP_OK;
}

tlp_status tlp_aggregate(tlp_graph g, const tlp_agg_desc *d, void *stream) {
    if (!d) return set_error(TLP_ERR_INVALID_ARGUMENT, "null descriptor");
    return aggregate(g, request_from_desc(*d), (cudaStream_t)stream);
}

tlp_status tlp_sage_aggregate(tlp_graph g, const float *X, int64_t F, int64_t ldx, int include_self,
                              float *Y, int64_t ldy, void *stream) {
    AggRequest r;
    r.op = OP_SAGE;
    r.X = X; r.F = F; r.ldx = ldx; r.Y = Y; r.ldy = ldy; r.sage_self = include_self ? 1 : 0;
    return aggregate(g, r, (cudaStream_t)stream);
}

tlp_status tlp_gat_mh_aggregate(tlp_graph g, const float *X, int64_t heads, int64_t F, int64_t ldx,
                                const float *el, const float *er, float slope, float *Y, int64_t ldy,
                                void *stream) {
    AggRequest r;
    r.op = OP_GATH;
    r.X = X; r.F = F; r.ldx = ldx; r.Y = Y; r.ldy = ldy;
    r.el = el; r.er = er; r.slope = slope; r.heads = heads;
    return aggregate(g, r, (cudaStream_t)stream);
}

}  // extern "C"

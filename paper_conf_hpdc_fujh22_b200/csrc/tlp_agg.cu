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
#include <cstdlib>
#include <cstring>

#include "tlp_internal.h"

namespace tlp {

// OP_SAGE: GraphSage mean (optionally with the self row); OP_GATH: multi-head
// GAT.
// OP_GATB: GAT backward on the transposed graph (NEXT-4, tlp_gat_backward).
enum Op : int { OP_GCN = 0, OP_GIN = 1, OP_GAT = 2, OP_SAGE = 3, OP_GATH = 4, OP_GATB = 5 };
enum Coef : int { COEF_NONE = 0, COEF_COUT = 1, COEF_W = 2, COEF_W_COUT = 3 };
enum Sched : int { S_DYNAMIC = 0, S_STATIC = 1, S_HARDWARE = 2 };

constexpr unsigned FULL = 0xffffffffu;

// Compile-time tuning knobs: source rows per
// gather group (two groups in flight per warp) and the launch bounds.
#ifndef TLP_U
#define TLP_U 2        // register path: rows per gather group (2 groups in flight)
#endif
#ifndef TLP_MAXT
#define TLP_MAXT 256   // threads per CTA at most (8 warps)
#endif
#ifndef TLP_MINB
#define TLP_MINB 3     // register path: 3 CTAs/SM -> <= 85 registers, 24 warps/SM
#endif
#ifndef TLP_MHB
#define TLP_MHB 4      // multi-head GAT: heads scored together per pass
#endif
#ifndef TLP_HINTS
#define TLP_HINTS 0    // 1: L2 evict_first policy on per-edge streams and Y stores (measured: no gain)
#endif
#ifndef TLP_MINB_LIGHT
#define TLP_MINB_LIGHT 4  // register path, no edge coefficient (GIN, SAGE): <= 64 registers, 32 warps/SM
#endif
#ifndef TLP_MINB_ASYNC
#define TLP_MINB_ASYNC 3  // async path: 3 CTAs/SM (ring = 3 x 64 KB of shared memory)
#endif

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
    int64_t ldx, ldy, ldp, row_offset, n_tasks, n_items, n_hubs, n_chunks, C;
    int F, n_strips, norm, step, sched, panel;
    int lps;  // lanes per strip (full-warp strips: lps * VEC columns, lps <= 32)
    float eps1, slope;
    int sage_self;  // OP_SAGE: include X[v] in the mean
    const float *bias;  // layer epilogue (NEXT-3): y = act(y + bias)
    int act;
    float act_param;
    int heads, fh;  // OP_GATH: H heads of fh columns each (F = heads * fh)
    // NEXT-2 fused all-gather: when n_dests > 0 every output row is stored to
    // dests[i] + (row_offset + r) * ldy for each destination (the Y_full of every
    // rank, mapped over NVLink) instead of to Y.
    float *const *dests;
    int n_dests;
    // hot-source L2 policy: when hot_thr != 0
    // colidx carries the source's out-degree class in bits 27-31; sources with
    // tag >= hot_thr are gathered with L2 evict_last, the rest with cold_first ?
    // evict_first : evict_normal.  A cache policy only: no value changes.
    unsigned hot_thr;
    int cold_first;
    // OP_GATB: forward X (the transposed row's own features) and the per-strip
    // edge dot products gbuf[s * gstride + e] = sum over strip s of
    // dY[v_e] . X[u] (transposed edge e).
    const float *xself;
    int64_t ldxs;
    // NEXT-3 epilogue projections: per strip s and local row r, the strip's
    // partial dots proj[(s * n_dst + r) * 2 + {0,1}] of the finished output
    // row with att_l / att_r (NULL proj: off)
    const float *att_l, *att_r;
    float *proj;
    int64_t n_dst;
    float *gbuf;
    int64_t gstride;
};

constexpr unsigned kIdxMask = (1u << 27) - 1u;

// Per-thread L2 policies for tagged gathers (createpolicy once per task).
struct GPol {
    unsigned thr;
    unsigned long long hot, cold;
};
__device__ __forceinline__ GPol make_gpol(const AggArgs &a) {
    GPol g;
    g.thr = a.hot_thr;
    g.hot = g.cold = 0;
    if (g.thr) {
        asm("createpolicy.fractional.L2::evict_last.b64 %0, 1.0;" : "=l"(g.hot));
        if (a.cold_first) asm("createpolicy.fractional.L2::evict_first.b64 %0, 1.0;" : "=l"(g.cold));
        else asm("createpolicy.fractional.L2::evict_normal.b64 %0, 1.0;" : "=l"(g.cold));
    }
    return g;
}

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
#if TLP_HINTS
        unsigned long long pol;
        asm("createpolicy.fractional.L2::evict_first.b64 %0, 1.0;" : "=l"(pol));
        asm volatile("st.global.L1::no_allocate.L2::cache_hint.v4.f32 [%0], {%1, %2, %3, %4}, %5;"
                     ::"l"(p), "f"(x.v[0]), "f"(x.v[1]), "f"(x.v[2]), "f"(x.v[3]), "l"(pol) : "memory");
#else
        *reinterpret_cast<float4 *>(p) = make_float4(x.v[0], x.v[1], x.v[2], x.v[3]);
#endif
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

// Gather address of source row u: base + u * row_bytes, one IMAD.WIDE.U32
// (32x32 -> 64-bit multiply-add); base = X + column (a byte pointer).
__device__ __forceinline__ const float *row_ptr(const char *base, unsigned u, unsigned row_bytes) {
    return reinterpret_cast<const float *>(base + (unsigned long long)u * row_bytes);
}

// ---- canonical reduction order ---------------------------------------------
// Every path reduces a row (or a hub chunk) as TWO interleaved chains: the
// edges at even and at odd positions (relative to the row / chunk start, in
// CSR order), each accumulated sequentially with fmaf, then added as
// even + odd.  Hub chunks start at even offsets (C is even) and are merged in
// chunk order.  The register path (full warp or half-warp PAIR), the cp.async
// path, every strip width, scheduler and partition produce exactly this
// order, hence bitwise-identical results.
//
// Lane -> edge mapping inside a 32-edge chunk, for step j, group slot k:
//   G = 1 (full warp): every lane gathers edge j+k for its 4 columns
//              (chain (j+k)&1);
//   G = 2 (PAIR): lanes 0-15 gather edge 2(j+k), lanes 16-31 edge 2(j+k)+1,
//              over 64 columns, so a warp-wide LDG.128 still moves 512 bytes
//              while the strip of X is half as wide (each half-warp is one
//              chain: the canonical even/odd order);
//   G = 4, 8 (narrow rows, F <= 32 / 16): lane group g = lane / (32/G) gathers
//              edge G(j+k)+g, so a warp instruction still moves G rows.  Group
//              g accumulates the chain of positions = g (mod G); the chains
//              are added by a fixed butterfly (xor 16, then 8, ...).  This
//              order depends only on F (never on P, the schedule or the
//              partition), so results stay bitwise reproducible and
//              partition-invariant; G <= 2 paths are bitwise identical to each
//              other (R10).

// Edge coefficients of lane-group gathers (G > 1) live in shared memory: the
// chunk's 32 coefficients are written once per chunk and read (broadcast) at
// consume time, so no coefficient register is held across the gather latency
// and the streamed-weight sums (GAT alpha mode, weighted GCN/GIN) fit 64
// registers, i.e. 4 CTAs / 32 warps per SM like the coefficient-free sums
// (measured: Reddit GAT 26.46 -> 24.42 ms, at 3 CTAs/SM 25.65 ms; GAT
// backward 36.3 -> 34.4 ms).
#ifndef TLP_SMEMC
#define TLP_SMEMC 1
#endif
#ifndef TLP_MINB_SMC
#define TLP_MINB_SMC 4   // resident CTAs for the shared-memory-coefficient kernels
#endif
__device__ __forceinline__ float *chunk_coef_smem() {
    __shared__ float tlp_cw[TLP_MAXT / 32][32];
    return tlp_cw[threadIdx.x >> 5];
}

template <int VEC, int U, bool HASC, int G, bool CLAMP, bool SMC = false>
__device__ __forceinline__ void issue_group(const char *base, unsigned row_bytes, int j, int n,
                                            int grp, int u_l, float c_l, Vec<VEC> (&xv)[U],
                                            float (&ck)[U]) {
#pragma unroll
    for (int k = 0; k < U; ++k) {
        int p = G * (j + k) + grp;
        if constexpr (CLAMP) p = min(p, n - 1);  // duplicate of a line in flight
        const unsigned u = (unsigned)__shfl_sync(FULL, u_l, p);
        if constexpr (HASC && !SMC) ck[k] = __shfl_sync(FULL, c_l, p);
        xv[k] = ld_vec<VEC>(row_ptr(base, u, row_bytes));
    }
}

// PHASE: parity of the group's first step (the caller's j is a multiple of 2U).
template <int VEC, int U, bool HASC, int G, bool GUARD, int PHASE, bool SMC = false>
__device__ __forceinline__ void consume_group(int j, int n, int grp, const Vec<VEC> (&xv)[U],
                                              const float (&ck)[U], Vec<VEC> (&ac)[2],
                                              const float *cw = nullptr) {
#pragma unroll
    for (int k = 0; k < U; ++k) {
        const int p = G * (j + k) + grp;
        const int ch = (G > 1) ? 0 : ((PHASE + k) & 1);
        if (!GUARD || p < n) {
            float cv = 0.f;
            if constexpr (HASC) cv = SMC ? cw[p] : ck[k];
#pragma unroll
            for (int c = 0; c < VEC; ++c) {
                if constexpr (HASC) ac[ch].v[c] = fmaf(cv, xv[k].v[c], ac[ch].v[c]);
                else ac[ch].v[c] += xv[k].v[c];
            }
        }
    }
}

// OP_GATB: per-edge dot products dY[v_e] . X[u] over this lane's columns,
// reduced across the lanes that share the edge (butterfly: the same bits in
// every lane); lane p keeps the dot of edge p of the chunk in g_l.
template <int VEC, int U, bool PAIR, bool GUARD>
__device__ __forceinline__ void dot_group(int j, int n, int lane, const Vec<VEC> (&xv)[U],
                                          const Vec<VEC> &xu, float &g_l) {
    const int half = PAIR ? (lane >> 4) : 0;
#pragma unroll
    for (int k = 0; k < U; ++k) {
        const int p = PAIR ? 2 * (j + k) + half : j + k;
        float d = 0.f;
#pragma unroll
        for (int c = 0; c < VEC; ++c) d = fmaf(xv[k].v[c], xu.v[c], d);
        if (GUARD && p >= n) d = 0.f;
        if constexpr (PAIR) {
#pragma unroll
            for (int o = 8; o > 0; o >>= 1) d += __shfl_xor_sync(FULL, d, o);
            const float other = __shfl_xor_sync(FULL, d, 16);
            const int t2 = 2 * (j + k);
            if (lane == t2) g_l = half == 0 ? d : other;
            if (lane == t2 + 1) g_l = half == 1 ? d : other;
        } else {
            d = warp_sum(d);
            if (lane == p) g_l = d;
        }
    }
}

// OP_GATB, full 32-edge chunks: the per-step lane partials are reduced by a
// streaming transposed butterfly.  Steps t are the gather steps of the chunk
// (PAIR: 16 steps of two edges, one per half-warp, 4 levels xor 8,4,2,1; full
// warp: 32 steps, 5 levels xor 16..1).  At level k a lane keeps the step whose
// bit matches its lane bit and adds its partner's partial of that step, so one
// shuffle reduces two steps; after the last level lane l holds the whole dot of
// step bitreverse(l) (PAIR: of edge 2*rev4(l & 15) + half).  15 (PAIR) or 31
// shuffles per 32 edges instead of 4-5 per edge.  t is a compile-time constant
// in the unrolled full-chunk loop, so the level logic folds away.
struct DotTree {
    float lv[5];
};
template <bool PAIR>
__device__ __forceinline__ void dot_push(DotTree &tr, float d, int t, int lane, float *gout) {
    constexpr int L = PAIR ? 4 : 5;
#pragma unroll
    for (int k = 0; k < L; ++k) {
        const int bitmask = (PAIR ? 8 : 16) >> k;  // lane bit of level k
        if (((t >> k) & 1) == 0) {  // first of the pair at this level: park it
            tr.lv[k] = d;
            return;
        }
        const bool hi = (lane & bitmask) != 0;
        const float keep = hi ? d : tr.lv[k];
        const float send = hi ? tr.lv[k] : d;
        d = keep + __shfl_xor_sync(FULL, send, bitmask);
    }
    // all levels done (t = last step): lane holds the dot of step rev(lane)
    const int l = PAIR ? (lane & 15) : lane;
    const int rv = PAIR ? (int)(__brev((unsigned)l) >> 28) : (int)(__brev((unsigned)l) >> 27);
    const int e = PAIR ? 2 * rv + (lane >> 4) : rv;
    gout[e] = d;
}
template <int VEC, int U, bool PAIR>
__device__ __forceinline__ void dot_tree(int j, int lane, const Vec<VEC> (&xv)[U],
                                         const Vec<VEC> &xu, DotTree &tr, float *gout) {
#pragma unroll
    for (int k = 0; k < U; ++k) {
        float d = 0.f;
#pragma unroll
        for (int c = 0; c < VEC; ++c) d = fmaf(xv[k].v[c], xu.v[c], d);
        dot_push<PAIR>(tr, d, j + k, lane, gout);
    }
}

// ---- L2 residency hints -------------------------------------------------------
// Per-edge streams (colidx, edge coefficients) and Y are touched once per strip:
// with TLP_HINTS they are loaded / stored with an L2 evict_first policy so they
// do not evict the L2-resident panel of X that every edge gathers from.
__device__ __forceinline__ unsigned long long policy_evict_first() {
    unsigned long long p;
    asm("createpolicy.fractional.L2::evict_first.b64 %0, 1.0;" : "=l"(p));
    return p;
}
__device__ __forceinline__ int ld_stream(const int32_t *ptr) {
#if TLP_HINTS
    int v;
    asm volatile("ld.global.nc.L1::no_allocate.L2::cache_hint.b32 %0, [%1], %2;"
                 : "=r"(v) : "l"(ptr), "l"(policy_evict_first()));
    return v;
#else
    return __ldg(ptr);
#endif
}
__device__ __forceinline__ float ld_stream(const float *ptr) {
#if TLP_HINTS
    float v;
    asm volatile("ld.global.nc.L1::no_allocate.L2::cache_hint.f32 %0, [%1], %2;"
                 : "=f"(v) : "l"(ptr), "l"(policy_evict_first()));
    return v;
#else
    return __ldg(ptr);
#endif
}

// Reduce the edges [e0, e1) of one destination row for the feature vector at
// `col` (a6 / a7).  GCN/GIN: acc = sum_e c_e X[u_e] (two-chain order above).
// GAT: online softmax state (m, den, acc = sum_e exp(s_e - m) X[u_e]).
//
// Latency hiding (the kernel is bound by bytes in flight, not by arithmetic):
//  * edge indices are loaded 32 at a time by the lanes two chunks ahead, and
//    the index-dependent values (c_out[u] or el[u]) one chunk ahead, so the
//    gathers of a chunk never wait on an index load;
//  * the gathers of a chunk are issued in double-buffered groups of U source
//    rows: the next group is in flight while the current one is accumulated;
//    full 32-edge chunks are fully unrolled (compile-time shuffle lanes).
template <int VEC, int OP, int COEF, int U, int G>
__device__ __forceinline__ void reduce_edges(const AggArgs &a, int64_t e0, int64_t e1,
                                             int col, bool active, float er_v, int lane,
                                             Vec<VEC> &acc, float &m, float &den,
                                             const Vec<VEC> &xu, float *gout) {
    // OP_GATB: the coefficient of transposed edge u -> v is alpha_e, streamed
    // (COEF_W) from the k_gatb_alpha pass; the strip's dot dY[v].X[u] of every
    // edge is reduced across lanes and stored to gout
    constexpr bool GB = (OP == OP_GATB);
    constexpr bool HASC = (COEF != COEF_NONE) || (OP == OP_GAT) || GB;
    constexpr bool DEP = (COEF & COEF_COUT) || (OP == OP_GAT);  // index-dependent value
    constexpr int STEPS = 32 / G;  // gather steps of a full chunk
    static_assert(STEPS % (2 * U) == 0, "U must divide the gather steps of a chunk in two groups");
    static_assert(!GB || G <= 2, "GAT backward edge dots: full warp or PAIR only");
    constexpr bool PAIR = (G == 2);
    constexpr bool SMC = TLP_SMEMC && HASC && (G > 1);
    float *cw = SMC ? chunk_coef_smem() : nullptr;
    // lanes past F read column 0 (a valid address); their results are never stored
    const char *base = reinterpret_cast<const char *>(a.X + (active ? col : 0));
    const unsigned row_bytes = (unsigned)a.ldx * 4u;
    const float *__restrict__ dep = (OP == OP_GAT) ? a.el : a.c_out;
    // 32-bit edge offsets relative to e0 (a row or hub chunk has < 2^31 edges)
    const int32_t *__restrict__ ci = a.colidx + e0;
    const float *__restrict__ wp = (COEF & COEF_W) ? a.ew + e0 : nullptr;
    const int len = (int)(e1 - e0);
    const int grp = lane / (32 / G);  // lane group (G > 1)
    Vec<VEC> ac[2];
#pragma unroll
    for (int c = 0; c < VEC; ++c) ac[0].v[c] = ac[1].v[c] = 0.f;
    if (len > 0) {
        int off = 0;
        int n0 = min(32, len);
        int n1 = min(32, len - 32);
        int u0 = 0, u1 = 0;
        float w0 = 1.f, w1 = 1.f, d0 = 0.f, d1 = 0.f;
        if (lane < n0) {
            u0 = ld_stream(ci + lane);
            if constexpr (COEF & COEF_W) w0 = ld_stream(wp + lane);
        }
        if (lane < n1) {
            u1 = ld_stream(ci + 32 + lane);
            if constexpr (COEF & COEF_W) w1 = ld_stream(wp + 32 + lane);
        }
        if constexpr (DEP)
            if (lane < n0) d0 = __ldg(dep + u0);
        while (true) {
            // two chunks ahead: indices; one chunk ahead: index-dependent values
            const int n2 = min(32, len - off - 64);
            int u2 = 0;
            float w2 = 1.f;
            if (lane < n2) {
                u2 = ld_stream(ci + off + 64 + lane);
                if constexpr (COEF & COEF_W) w2 = ld_stream(wp + off + 64 + lane);
            }
            if constexpr (DEP)
                if (lane < n1) d1 = __ldg(dep + u1);
            // coefficients of the current chunk
            float c_l = 1.f;
            if constexpr (OP == OP_GAT) {
                float s = -INFINITY;
                if (lane < n0) {
                    const float t = d0 + er_v;
                    s = t >= 0.f ? t : a.slope * t;  // LeakyReLU (R6)
                }
                const float m_new = fmaxf(m, warp_max(s));
                const float scale = __expf(m - m_new);  // m = -inf -> 0
                c_l = (lane < n0) ? __expf(s - m_new) : 0.f;
                den = fmaf(den, scale, warp_sum(c_l));
#pragma unroll
                for (int c = 0; c < VEC; ++c) {
                    ac[0].v[c] *= scale;
                    ac[1].v[c] *= scale;
                }
                m = m_new;
            } else {
                if constexpr (COEF & COEF_COUT) c_l = d0;
                if constexpr (COEF & COEF_W) c_l *= w0;
            }
            if constexpr (SMC) {
                __syncwarp();  // the previous chunk's coefficients are consumed
                cw[lane] = c_l;
                __syncwarp();
            }
            Vec<VEC> xa[U], xb[U];
            float ca[U], cb[U];
            float g_l = 0.f;  // OP_GATB (partial chunk): this strip's dot of edge `lane`
            DotTree dt_;      // OP_GATB (full chunk): pending butterfly levels
            if (n0 == 32) {
                // full chunk: fully unrolled, compile-time shuffle lanes, no guards
                issue_group<VEC, U, HASC, G, false, SMC>(base, row_bytes, 0, 32, grp, u0, c_l, xa, ca);
#pragma unroll
                for (int j = 0; j < STEPS; j += 2 * U) {
                    issue_group<VEC, U, HASC, G, false, SMC>(base, row_bytes, j + U, 32, grp, u0, c_l, xb, cb);
                    consume_group<VEC, U, HASC, G, false, 0, SMC>(j, 32, grp, xa, ca, ac, cw);
                    if constexpr (GB) dot_tree<VEC, U, PAIR>(j, lane, xa, xu, dt_, gout + off);
                    if (j + 2 * U < STEPS)
                        issue_group<VEC, U, HASC, G, false, SMC>(base, row_bytes, j + 2 * U, 32, grp, u0, c_l, xa, ca);
                    consume_group<VEC, U, HASC, G, false, U, SMC>(j + U, 32, grp, xb, cb, ac, cw);
                    if constexpr (GB) dot_tree<VEC, U, PAIR>(j + U, lane, xb, xu, dt_, gout + off);
                }
            } else {
                // partial chunk (n0 is warp-uniform: the guards never diverge)
                const int steps = (n0 + G - 1) / G;
                issue_group<VEC, U, HASC, G, true, SMC>(base, row_bytes, 0, n0, grp, u0, c_l, xa, ca);
                for (int j = 0; j < steps; j += 2 * U) {
                    const bool more = j + U < steps;
                    if (more) issue_group<VEC, U, HASC, G, true, SMC>(base, row_bytes, j + U, n0, grp, u0, c_l, xb, cb);
                    consume_group<VEC, U, HASC, G, true, 0, SMC>(j, n0, grp, xa, ca, ac, cw);
                    if constexpr (GB) dot_group<VEC, U, PAIR, true>(j, n0, lane, xa, xu, g_l);
                    if (j + 2 * U < steps)
                        issue_group<VEC, U, HASC, G, true, SMC>(base, row_bytes, j + 2 * U, n0, grp, u0, c_l, xa, ca);
                    if (more) consume_group<VEC, U, HASC, G, true, U, SMC>(j + U, n0, grp, xb, cb, ac, cw);
                    if constexpr (GB)
                        if (more) dot_group<VEC, U, PAIR, true>(j + U, n0, lane, xb, xu, g_l);
                }
            }
            if constexpr (GB)
                if (n0 < 32 && lane < n0) gout[off + lane] = g_l;  // partial chunk
            if (n1 <= 0) break;
            off += 32;
            n0 = n1; n1 = n2;
            u0 = u1; u1 = u2;
            w0 = w1; w1 = w2;
            d0 = d1;
        }
    }
    // even + odd (G = 2: the odd chain lives in the other half-warp); G > 2:
    // the group chains added by a fixed butterfly
#pragma unroll
    for (int c = 0; c < VEC; ++c) {
        if constexpr (G > 1) {
            float x = ac[0].v[c];
#pragma unroll
            for (int o = 16; o >= 32 / G; o >>= 1) x += __shfl_xor_sync(FULL, x, o);
            acc.v[c] = x;
        } else {
            acc.v[c] = ac[0].v[c] + ac[1].v[c];
        }
    }
}

// ---- asynchronous-copy path ------------------------------------------------
// The gathered rows land in a per-warp shared-memory ring through cp.async
// (LDGSTS, L2 -> SMEM, bypassing L1 and the register file), D edges deep.  Bytes
// in flight then cost no registers, so occupancy and depth are decoupled.
#ifndef TLP_DEPTH
#define TLP_DEPTH 16   // edges in flight per warp on the async path
#endif

template <int VEC>
__device__ __forceinline__ void cp_async_vec(float *dst_smem, const float *src, bool pred) {
    const unsigned d = (unsigned)__cvta_generic_to_shared(dst_smem);
    const int bytes = pred ? 4 * VEC : 0;  // src-size 0 => zero fill, no global read
    if constexpr (VEC == 4)
        asm volatile("cp.async.cg.shared.global [%0], [%1], 16, %2;\n" ::"r"(d), "l"(src), "r"(bytes));
    else if constexpr (VEC == 2)
        asm volatile("cp.async.ca.shared.global [%0], [%1], 8, %2;\n" ::"r"(d), "l"(src), "r"(bytes));
    else
        asm volatile("cp.async.ca.shared.global [%0], [%1], 4, %2;\n" ::"r"(d), "l"(src), "r"(bytes));
}
// cp.async of source row u (possibly tagged) with the hot/cold L2 policy.
template <int VEC>
__device__ __forceinline__ void cp_async_x(float *dst_smem, const char *base, unsigned u,
                                           unsigned row_bytes, const GPol &gp, bool pred) {
    const float *src = reinterpret_cast<const float *>(
        base + (unsigned long long)(u & kIdxMask) * row_bytes);
    if (gp.thr == 0 || VEC != 4) {
        cp_async_vec<VEC>(dst_smem, src, pred);
        return;
    }
    const unsigned d = (unsigned)__cvta_generic_to_shared(dst_smem);
    const int bytes = pred ? 16 : 0;
    const unsigned long long pol = u >= gp.thr ? gp.hot : gp.cold;
    asm volatile("cp.async.cg.shared.global.L2::cache_hint [%0], [%1], 16, %2, %3;\n"
                 ::"r"(d), "l"(src), "r"(bytes), "l"(pol));
}
__device__ __forceinline__ void cp_async_commit() { asm volatile("cp.async.commit_group;\n" ::); }
template <int N>
__device__ __forceinline__ void cp_async_wait() { asm volatile("cp.async.wait_group %0;\n" ::"n"(N)); }

template <int VEC>
__device__ __forceinline__ float *warp_ring() {
    extern __shared__ __align__(16) float tlp_smem[];
    const int w = threadIdx.x >> 5;
    return tlp_smem + (size_t)w * TLP_DEPTH * 32 * VEC;
}

template <int VEC, bool HASC>
__device__ __forceinline__ void acc_from_smem(const float *src, float cj, Vec<VEC> &acc) {
    if constexpr (VEC == 4) {
        const float4 x = *reinterpret_cast<const float4 *>(src);
        if constexpr (HASC) {
            acc.v[0] = fmaf(cj, x.x, acc.v[0]); acc.v[1] = fmaf(cj, x.y, acc.v[1]);
            acc.v[2] = fmaf(cj, x.z, acc.v[2]); acc.v[3] = fmaf(cj, x.w, acc.v[3]);
        } else {
            acc.v[0] += x.x; acc.v[1] += x.y; acc.v[2] += x.z; acc.v[3] += x.w;
        }
    } else {
#pragma unroll
        for (int c = 0; c < VEC; ++c) {
            if constexpr (HASC) acc.v[c] = fmaf(cj, src[c], acc.v[c]);
            else acc.v[c] += src[c];
        }
    }
}

template <int VEC, int OP, int COEF, int U>
__device__ __forceinline__ void reduce_edges_async(const AggArgs &a, int64_t e0, int64_t e1,
                                                   int col, bool active, float er_v, int lane,
                                                   Vec<VEC> &acc, float &m, float &den) {
    constexpr int D = TLP_DEPTH;
    constexpr bool HASC = (COEF != COEF_NONE) || (OP == OP_GAT);
    constexpr bool DEP = (COEF & COEF_COUT) || (OP == OP_GAT);
    const char *base = reinterpret_cast<const char *>(a.X + (active ? col : 0));
    const unsigned row_bytes = (unsigned)a.ldx * 4u;
    const float *__restrict__ dep = (OP == OP_GAT) ? a.el : a.c_out;
    const GPol gp = make_gpol(a);
    const int32_t *__restrict__ ci = a.colidx + e0;
    const float *__restrict__ wp = (COEF & COEF_W) ? a.ew + e0 : nullptr;
    const int len = (int)(e1 - e0);
    Vec<VEC> ae, ao;  // even / odd chains (canonical order)
#pragma unroll
    for (int c = 0; c < VEC; ++c) ae.v[c] = ao.v[c] = 0.f;
    if (len > 0) {
        float *ring = warp_ring<VEC>() + lane * VEC;
        int off = 0;
        int n0 = min(32, len);
        int n1 = min(32, len - 32);
        int u0 = 0, u1 = 0;
        float w0 = 1.f, w1 = 1.f, d0 = 0.f, d1 = 0.f;
        if (lane < n0) {
            u0 = ld_stream(ci + lane);
            if constexpr (COEF & COEF_W) w0 = ld_stream(wp + lane);
        }
        if (lane < n1) {
            u1 = ld_stream(ci + 32 + lane);
            if constexpr (COEF & COEF_W) w1 = ld_stream(wp + 32 + lane);
        }
        if constexpr (DEP)
            if (lane < n0) d0 = __ldg(dep + (u0 & kIdxMask));
        // prologue: edges 0 .. D-2 in flight
#pragma unroll
        for (int k = 0; k < D - 1; ++k) {
            const int uk = __shfl_sync(FULL, k < 32 ? u0 : u1, k & 31);
            cp_async_x<VEC>(ring + k * 32 * VEC, base, (unsigned)uk, row_bytes, gp, active && k < len);
            cp_async_commit();
        }
        int slot = 0;  // ring slot of edge `off + j`
        while (true) {
            const int n2 = min(32, len - off - 64);
            int u2 = 0;
            float w2 = 1.f;
            if (lane < n2) {
                u2 = ld_stream(ci + off + 64 + lane);
                if constexpr (COEF & COEF_W) w2 = ld_stream(wp + off + 64 + lane);
            }
            if constexpr (DEP)
                if (lane < n1) d1 = __ldg(dep + (u1 & kIdxMask));
            float c_l = 1.f;
            if constexpr (OP == OP_GAT) {
                float s = -INFINITY;
                if (lane < n0) {
                    const float t = d0 + er_v;
                    s = t >= 0.f ? t : a.slope * t;
                }
                const float m_new = fmaxf(m, warp_max(s));
                const float scale = __expf(m - m_new);
                c_l = (lane < n0) ? __expf(s - m_new) : 0.f;
                den = fmaf(den, scale, warp_sum(c_l));
#pragma unroll
                for (int c = 0; c < VEC; ++c) {
                    ae.v[c] *= scale;
                    ao.v[c] *= scale;
                }
                m = m_new;
            } else {
                if constexpr (COEF & COEF_COUT) c_l = d0;
                if constexpr (COEF & COEF_W) c_l *= w0;
            }
            for (int j = 0; j < n0; ++j) {
                // issue edge j + D - 1 (in this chunk or the next one)
                const int jj = j + D - 1;
                const int ui = __shfl_sync(FULL, jj < 32 ? u0 : u1, jj & 31);
                const bool valid = (off + jj) < len;
                int ws = slot + D - 1;
                if (ws >= D) ws -= D;
                cp_async_x<VEC>(ring + ws * 32 * VEC, base, (unsigned)ui, row_bytes, gp, active && valid);
                cp_async_commit();
                cp_async_wait<D - 1>();
                const float cj = __shfl_sync(FULL, c_l, j);
                // chunks start at even offsets: the parity of j is the edge's parity
                if (j & 1) acc_from_smem<VEC, HASC>(ring + slot * 32 * VEC, cj, ao);
                else acc_from_smem<VEC, HASC>(ring + slot * 32 * VEC, cj, ae);
                if (++slot == D) slot = 0;
            }
            if (n1 <= 0) break;
            off += 32;
            n0 = n1; n1 = n2;
            u0 = u1; u1 = u2;
            w0 = w1; w1 = w2;
            d0 = d1;
        }
        cp_async_wait<0>();  // drain the (empty) tail groups before the ring is reused
    }
#pragma unroll
    for (int c = 0; c < VEC; ++c) acc.v[c] = ae.v[c] + ao.v[c];
}

// ---- multi-head GAT (NEXT-1) -----------------------------------------------
// Head h owns columns [h*fh, (h+1)*fh) (fh a multiple of VEC, so a lane's
// vector lies in one head).  A strip of 32*VEC columns spans heads
// [h_lo, h_lo+nh).  Per 32-edge chunk the warp computes, head by head, the
// LeakyReLU scores, the online-softmax update (running max M, denominator D,
// rescale S) and the weights p[j], kept in a per-warp shared-memory block;
// each lane then gathers with the weights of its own head.  Scores never
// leave the SM.  Reduction order: the canonical two chains per head.
constexpr int kMhMaxHeads = 33;  // heads one strip can touch (fh >= VEC)
constexpr int kMhWarpFloats = kMhMaxHeads * 32 + 3 * kMhMaxHeads + 1;  // P, M, D, S (+pad)

__device__ __forceinline__ float *mh_warp_smem() {
    extern __shared__ __align__(16) float tlp_smem[];
    return tlp_smem + (size_t)(threadIdx.x >> 5) * kMhWarpFloats;
}

// Scores, online-softmax update and weights of one 32-edge chunk for the heads
// [h_lo, h_lo+nh) of a strip (lane j holds edge j with source u_l).  Heads are
// processed TLP_MHB at a time so their el loads and warp reductions overlap.
__device__ __forceinline__ void mh_chunk_scores(const AggArgs &a, int u_l, int n0, int H, int h_lo,
                                                int nh, const float *__restrict__ erv, int lane,
                                                float *P, float *M, float *D, float *S) {
    constexpr int B = TLP_MHB;
    const float *__restrict__ elu = a.el + (size_t)((unsigned)u_l) * H + h_lo;
    for (int hb = 0; hb < nh; hb += B) {
        float sv[B], mo[B], mn[B], sm[B];
#pragma unroll
        for (int k = 0; k < B; ++k) {
            sv[k] = -INFINITY;
            if (hb + k < nh && lane < n0) {
                const float t = __ldg(elu + hb + k) + __ldg(erv + hb + k);
                sv[k] = t >= 0.f ? t : a.slope * t;  // LeakyReLU (R6)
            }
        }
#pragma unroll
        for (int k = 0; k < B; ++k) {
            if (hb + k < nh) {  // warp-uniform
                mo[k] = M[hb + k];
                mn[k] = fmaxf(mo[k], warp_max(sv[k]));
                const float p = (lane < n0) ? __expf(sv[k] - mn[k]) : 0.f;
                sm[k] = warp_sum(p);
                P[(hb + k) * 32 + lane] = p;
            }
        }
        __syncwarp();
        if (lane == 0) {
#pragma unroll
            for (int k = 0; k < B; ++k)
                if (hb + k < nh) {
                    const float scale = __expf(mo[k] - mn[k]);
                    M[hb + k] = mn[k];
                    D[hb + k] = fmaf(D[hb + k], scale, sm[k]);
                    S[hb + k] = scale;
                }
        }
        __syncwarp();
    }
}

// A lane's VEC columns [col, col+VEC) lie in at most two heads (fh >= VEC):
// head slot hl for components c < split, hl + 1 for the rest.
template <int VEC, int U>
__device__ __forceinline__ void reduce_edges_mh(const AggArgs &a, int64_t e0, int64_t e1, int s,
                                                int col, bool active, int64_t rglob, int lane,
                                                Vec<VEC> &acc, float *&Mh, float *&Dh, int &h_lo,
                                                int &nh, int &hl, int &split) {
    float *P = mh_warp_smem();
    float *M = P + kMhMaxHeads * 32;
    float *D = M + kMhMaxHeads;
    float *S = D + kMhMaxHeads;
    Mh = M;
    Dh = D;
    const int H = a.heads, fh = a.fh;
    const int c_lo = s * 32 * VEC;
    const int c_hi = min(a.F, c_lo + 32 * VEC) - 1;
    h_lo = c_lo / fh;
    nh = c_hi / fh - h_lo + 1;
    const int cc = active ? col : c_lo;
    hl = cc / fh - h_lo;
    split = (hl + h_lo + 1) * fh - cc;                 // components in head hl
    const int hl2 = min(hl + (split < VEC ? 1 : 0), nh - 1);
    for (int hh = lane; hh < nh; hh += 32) {
        M[hh] = -INFINITY;
        D[hh] = 0.f;
    }
    __syncwarp();
    const char *base = reinterpret_cast<const char *>(a.X + (active ? col : 0));
    const unsigned row_bytes = (unsigned)a.ldx * 4u;
    const int32_t *__restrict__ ci = a.colidx + e0;
    const float *__restrict__ erv = a.er + rglob * H + h_lo;
    const int len = (int)(e1 - e0);
    Vec<VEC> ac[2];
#pragma unroll
    for (int c = 0; c < VEC; ++c) ac[0].v[c] = ac[1].v[c] = 0.f;
    for (int off = 0; off < len; off += 32) {
        const int n0 = min(32, len - off);
        const int u_l = (lane < n0) ? __ldg(ci + off + lane) : 0;
        mh_chunk_scores(a, u_l, n0, H, h_lo, nh, erv, lane, P, M, D, S);
        const float sA = S[hl], sB = S[hl2];
#pragma unroll
        for (int c = 0; c < VEC; ++c) {
            const float sc = (c < split) ? sA : sB;
            ac[0].v[c] *= sc;
            ac[1].v[c] *= sc;
        }
        const float *pa = P + hl * 32;
        const float *pb = P + hl2 * 32;
        for (int j = 0; j < n0; j += 2 * U) {
            Vec<VEC> xv[2 * U];
            float ca[2 * U], cb[2 * U];
#pragma unroll
            for (int k = 0; k < 2 * U; ++k) {
                const int jj = min(j + k, n0 - 1);
                const unsigned u = (unsigned)__shfl_sync(FULL, u_l, jj);
                ca[k] = pa[jj];
                cb[k] = pb[jj];
                xv[k] = ld_vec<VEC>(row_ptr(base, u, row_bytes));
            }
#pragma unroll
            for (int k = 0; k < 2 * U; ++k)
                if (j + k < n0) {
#pragma unroll
                    for (int c = 0; c < VEC; ++c)
                        ac[k & 1].v[c] = fmaf(c < split ? ca[k] : cb[k], xv[k].v[c], ac[k & 1].v[c]);
                }
        }
        __syncwarp();  // P, S are rewritten by the next chunk
    }
#pragma unroll
    for (int c = 0; c < VEC; ++c) acc.v[c] = ac[0].v[c] + ac[1].v[c];
}

// Multi-head GAT with the cp.async ring (gathers that stream from HBM): the
// per-warp shared memory holds the head block followed by a D-deep ring.
template <int VEC>
__device__ __forceinline__ float *mh_warp_ring() {
    extern __shared__ __align__(16) float tlp_smem[];
    constexpr int stride = kMhWarpFloats + TLP_DEPTH * 32 * VEC;
    return tlp_smem + (size_t)(threadIdx.x >> 5) * stride + kMhWarpFloats;
}
template <int VEC>
__device__ __forceinline__ float *mh_warp_smem_async() {
    extern __shared__ __align__(16) float tlp_smem[];
    constexpr int stride = kMhWarpFloats + TLP_DEPTH * 32 * VEC;
    return tlp_smem + (size_t)(threadIdx.x >> 5) * stride;
}

template <int VEC>
__device__ __forceinline__ void reduce_edges_mh_async(const AggArgs &a, int64_t e0, int64_t e1,
                                                      int s, int col, bool active, int64_t rglob,
                                                      int lane, Vec<VEC> &acc, float *&Mh,
                                                      float *&Dh, int &h_lo, int &nh, int &hl,
                                                      int &split) {
    constexpr int DD = TLP_DEPTH;
    float *P = mh_warp_smem_async<VEC>();
    float *M = P + kMhMaxHeads * 32;
    float *Dn = M + kMhMaxHeads;
    float *S = Dn + kMhMaxHeads;
    Mh = M;
    Dh = Dn;
    const int H = a.heads, fh = a.fh;
    const int c_lo = s * 32 * VEC;
    const int c_hi = min(a.F, c_lo + 32 * VEC) - 1;
    h_lo = c_lo / fh;
    nh = c_hi / fh - h_lo + 1;
    const int cc = active ? col : c_lo;
    hl = cc / fh - h_lo;
    split = (hl + h_lo + 1) * fh - cc;
    const int hl2 = min(hl + (split < VEC ? 1 : 0), nh - 1);
    for (int hh = lane; hh < nh; hh += 32) {
        M[hh] = -INFINITY;
        Dn[hh] = 0.f;
    }
    __syncwarp();
    const char *base = reinterpret_cast<const char *>(a.X + (active ? col : 0));
    const unsigned row_bytes = (unsigned)a.ldx * 4u;
    const int32_t *__restrict__ ci = a.colidx + e0;
    const float *__restrict__ erv = a.er + rglob * H + h_lo;
    const int len = (int)(e1 - e0);
    Vec<VEC> ae, ao;
#pragma unroll
    for (int c = 0; c < VEC; ++c) ae.v[c] = ao.v[c] = 0.f;
    if (len > 0) {
        float *ring = mh_warp_ring<VEC>() + lane * VEC;
        int n0 = min(32, len), n1 = min(32, len - 32);
        int u0 = (lane < n0) ? __ldg(ci + lane) : 0;
        int u1 = (lane < n1) ? __ldg(ci + 32 + lane) : 0;
#pragma unroll
        for (int k = 0; k < DD - 1; ++k) {
            const int uk = __shfl_sync(FULL, k < 32 ? u0 : u1, k & 31);
            cp_async_vec<VEC>(ring + k * 32 * VEC, row_ptr(base, (unsigned)uk, row_bytes), active && k < len);
            cp_async_commit();
        }
        int slot = 0, off = 0;
        while (true) {
            const int n2 = min(32, len - off - 64);
            const int u2 = (lane < n2) ? __ldg(ci + off + 64 + lane) : 0;
            mh_chunk_scores(a, u0, n0, H, h_lo, nh, erv, lane, P, M, Dn, S);
            const float sA = S[hl], sB = S[hl2];
#pragma unroll
            for (int c = 0; c < VEC; ++c) {
                const float sc = (c < split) ? sA : sB;
                ae.v[c] *= sc;
                ao.v[c] *= sc;
            }
            const float *pa = P + hl * 32;
            const float *pb = P + hl2 * 32;
            for (int j = 0; j < n0; ++j) {
                const int jj = j + DD - 1;
                const int ui = __shfl_sync(FULL, jj < 32 ? u0 : u1, jj & 31);
                int ws = slot + DD - 1;
                if (ws >= DD) ws -= DD;
                cp_async_vec<VEC>(ring + ws * 32 * VEC, row_ptr(base, (unsigned)ui, row_bytes),
                                  active && (off + jj) < len);
                cp_async_commit();
                cp_async_wait<DD - 1>();
                const float ca = pa[j], cb = pb[j];
                const float *src = ring + slot * 32 * VEC;
                Vec<VEC> &ac = (j & 1) ? ao : ae;
#pragma unroll
                for (int c = 0; c < VEC; ++c) ac.v[c] = fmaf(c < split ? ca : cb, src[c], ac.v[c]);
                if (++slot == DD) slot = 0;
            }
            __syncwarp();  // P, S are rewritten by the next chunk
            if (n1 <= 0) break;
            off += 32;
            n0 = n1; n1 = n2;
            u0 = u1; u1 = u2;
        }
        cp_async_wait<0>();
    }
#pragma unroll
    for (int c = 0; c < VEC; ++c) acc.v[c] = ae.v[c] + ao.v[c];
}

// Layer epilogue (NEXT-3, Eq. 2): y = act(y + bias), per element, so it never
// changes with strip width or gather path.
template <int VEC>
__device__ __forceinline__ void apply_layer_epilogue(const AggArgs &a, int col, Vec<VEC> &y) {
    if (a.bias) {
#pragma unroll
        for (int c = 0; c < VEC; ++c)
            if (col + c < a.F) y.v[c] += __ldg(a.bias + col + c);
    }
    if (a.act == TLP_ACT_RELU) {
#pragma unroll
        for (int c = 0; c < VEC; ++c) y.v[c] = y.v[c] > 0.f ? y.v[c] : 0.f;
    } else if (a.act == TLP_ACT_LEAKY_RELU) {
#pragma unroll
        for (int c = 0; c < VEC; ++c) y.v[c] = y.v[c] >= 0.f ? y.v[c] : a.act_param * y.v[c];
    } else if (a.act == TLP_ACT_ELU) {
#pragma unroll
        for (int c = 0; c < VEC; ++c) y.v[c] = y.v[c] > 0.f ? y.v[c] : a.act_param * expm1f(y.v[c]);
    }
}

// Epilogue (a9) for a full row reduction.
template <int VEC, int OP>
__device__ __forceinline__ Vec<VEC> epilogue(const AggArgs &a, int64_t r, int64_t deg, int col,
                                             bool active, const Vec<VEC> &acc, float den) {
    Vec<VEC> y;
    if constexpr (OP == OP_GATB) {
        y = acc;  // dX[u] = sum_e alpha_e dY[v_e]
    } else if constexpr (OP == OP_GCN) {
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
    } else if constexpr (OP == OP_SAGE) {
        // mean over N(v) (+ v itself when sage_self): (X[v] + sum) / (deg + 1)
        const int64_t cnt = deg + a.sage_self;
        const float inv = 1.0f / (float)(cnt > 1 ? cnt : 1);
        Vec<VEC> xs;
#pragma unroll
        for (int c = 0; c < VEC; ++c) xs.v[c] = 0.f;
        if (a.sage_self && active) xs = ld_vec<VEC>(a.X + (a.row_offset + r) * a.ldx + col);
#pragma unroll
        for (int c = 0; c < VEC; ++c) y.v[c] = (xs.v[c] + acc.v[c]) * inv;
    } else {
#pragma unroll
        for (int c = 0; c < VEC; ++c) y.v[c] = deg > 0 ? acc.v[c] / den : 0.f;
    }
    apply_layer_epilogue<VEC>(a, col, y);
    return y;
}

// Store a finished output vector of local row r: to Y, or (fused all-gather)
// to the same global row of every destination buffer.
template <int VEC>
__device__ __forceinline__ void store_out(const AggArgs &a, int64_t r, int col, const Vec<VEC> &y) {
    if (a.n_dests == 0) {
        st_row<VEC>(a.Y + r * a.ldy, col, a.F, y);
    } else {
        const int64_t off = (a.row_offset + r) * a.ldy;
        for (int i = 0; i < a.n_dests; ++i) st_row<VEC>(a.dests[i] + off, col, a.F, y);
    }
}

// Column of this lane's vector in strip s (G > 1: strips of 32/G lanes x VEC
// columns, lanes l and l + 32/G share a column; PAIR = 64-column strips), and
// whether this lane stores it.
template <int VEC, int G>
__device__ __forceinline__ int strip_col(const AggArgs &a, int s, int lane) {
    constexpr int LG = 32 / G;
    return (G > 1) ? s * LG * VEC + (lane % LG) * VEC : s * a.lps * VEC + lane * VEC;
}
// Whether this lane's column of the strip exists (narrow strips leave lanes
// >= lps idle; they gather column 0 of the same row, a sector already fetched).
template <int G>
__device__ __forceinline__ bool in_strip(const AggArgs &a, int lane, int col) {
    return (G > 1 || lane < a.lps) && col < a.F;
}
template <int G>
__device__ __forceinline__ bool stores(int lane) {
    return G == 1 || lane < 32 / G;
}

// NEXT-3: the strip's partial dots of a finished row vector with att_l, att_r
// (per-lane fma over the vector, butterfly over the warp; lane 0 stores).
template <int VEC, int G>
__device__ __forceinline__ void project_row(const AggArgs &a, int64_t r, int s, int col, bool active,
                                            const Vec<VEC> &y, int lane) {
    if (a.proj == nullptr) return;
    float pl = 0.f, pr = 0.f;
    if (active && stores<G>(lane)) {
#pragma unroll
        for (int c = 0; c < VEC; ++c) {
            if (col + c < a.F) {
                if (a.att_l) pl = fmaf(y.v[c], __ldg(a.att_l + col + c), pl);
                if (a.att_r) pr = fmaf(y.v[c], __ldg(a.att_r + col + c), pr);
            }
        }
    }
    pl = warp_sum(pl);
    pr = warp_sum(pr);
    if (lane == 0) {
        float *p = a.proj + ((int64_t)s * a.n_dst + r) * 2;
        p[0] = pl;
        p[1] = pr;
    }
}


// OP_GATB: the transposed row's own forward features X[u] for this lane's
// columns of strip s, and where the strip's edge dot products go.
template <int VEC, int OP>
__device__ __forceinline__ void gatb_self(const AggArgs &a, int64_t r, int s, int64_t e0, int col,
                                          bool active, Vec<VEC> &xu, float *&gout) {
#pragma unroll
    for (int c = 0; c < VEC; ++c) xu.v[c] = 0.f;
    if constexpr (OP == OP_GATB) {
        if (active) xu = ld_vec<VEC>(a.xself + r * a.ldxs + col);
        gout = a.gbuf + (int64_t)s * a.gstride + e0;
    }
}

// A regular work unit: whole rows [r0, r1), feature strips [s0, s1).
template <int VEC, int OP, int COEF, int U, bool ASYNC, int G>
__device__ __forceinline__ void do_unit(const AggArgs &a, int r0, int r1, int s0, int s1,
                                        int lane) {
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
            for (int s = s0; s < s1; ++s) {
                const int col = strip_col<VEC, G>(a, s, lane);
                const bool active = in_strip<G>(a, lane, col);
                Vec<VEC> acc;
#pragma unroll
                for (int c = 0; c < VEC; ++c) acc.v[c] = 0.f;
                float m = -INFINITY, den = 0.f;
                if constexpr (OP == OP_GATH) {
                    float *Mh, *Dh;
                    int h_lo, nh, hl, split;
                    if constexpr (ASYNC)
                        reduce_edges_mh_async<VEC>(a, e0, e1, s, col, active, a.row_offset + r, lane,
                                                   acc, Mh, Dh, h_lo, nh, hl, split);
                    else
                        reduce_edges_mh<VEC, U>(a, e0, e1, s, col, active, a.row_offset + r, lane, acc,
                                                Mh, Dh, h_lo, nh, hl, split);
                    const float dA = Dh[hl], dB = Dh[min(hl + 1, nh - 1)];
                    __syncwarp();  // the head state is reset by the next strip / row
                    Vec<VEC> y;
#pragma unroll
                    for (int c = 0; c < VEC; ++c)
                        y.v[c] = (e1 > e0) ? acc.v[c] / (c < split ? dA : dB) : 0.f;
                    apply_layer_epilogue<VEC>(a, col, y);
                    if (active) store_out<VEC>(a, r, col, y);
                    continue;
                } else if constexpr (ASYNC) {
                    reduce_edges_async<VEC, OP, COEF, U>(a, e0, e1, col, active, er_v, lane, acc, m, den);
                } else {
                    Vec<VEC> xu;
                    float *gout = nullptr;
                    gatb_self<VEC, OP>(a, r, s, e0, col, active, xu, gout);
                    reduce_edges<VEC, OP, COEF, U, G>(a, e0, e1, col, active, er_v, lane, acc, m, den,
                                                         xu, gout);
                }
                Vec<VEC> y = epilogue<VEC, OP>(a, r, e1 - e0, col, active, acc, den);
                if (active && stores<G>(lane)) store_out<VEC>(a, r, col, y);
                project_row<VEC, G>(a, r, s, col, active, y, lane);
            }
        }
    }
}

// One C-edge chunk of hub h (a8), feature strips [s0, s1).  The last chunk of
// the hub to finish these strips merges all its partials in chunk order and
// writes the row.  Tickets (and GAT (m, den) pairs) are kept per panel s0.
template <int VEC, int OP, int COEF, int U, bool ASYNC, int G>
__device__ __forceinline__ void do_hub_chunk(const AggArgs &a, int h, int j, int s0, int s1,
                                             int lane) {
    const int r = __ldg(a.hub_row + h);
    const int off = __ldg(a.hub_off + h);
    const int nch = __ldg(a.hub_off + h + 1) - off;
    const int64_t eb = __ldg(a.rowptr + r), ee = __ldg(a.rowptr + r + 1);
    const int64_t e0 = eb + (int64_t)j * a.C;
    const int64_t e1 = min(e0 + a.C, ee);
    float er_v = 0.f;
    if constexpr (OP == OP_GAT) er_v = __ldg(a.er + a.row_offset + r);
    const int slot = off + j;
    // this panel's (m, den) pairs: [n_chunks][heads] (heads = 1 unless OP_GATH)
    const int mdh = (OP == OP_GATH) ? a.heads : 1;
    float *md = a.md + 2 * (int64_t)s0 * a.n_chunks * mdh;
    int32_t *ticket = a.hub_ticket + (int64_t)s0 * a.n_hubs + h;
    for (int s = s0; s < s1; ++s) {
        const int col = strip_col<VEC, G>(a, s, lane);
        const bool active = in_strip<G>(a, lane, col);
        Vec<VEC> acc;
#pragma unroll
        for (int c = 0; c < VEC; ++c) acc.v[c] = 0.f;
        float m = -INFINITY, den = 0.f;
        if constexpr (OP == OP_GATH) {
            float *Mh, *Dh;
            int h_lo, nh, hl, split;
            if constexpr (ASYNC)
                reduce_edges_mh_async<VEC>(a, e0, e1, s, col, active, a.row_offset + r, lane, acc, Mh,
                                           Dh, h_lo, nh, hl, split);
            else
                reduce_edges_mh<VEC, U>(a, e0, e1, s, col, active, a.row_offset + r, lane, acc, Mh, Dh,
                                        h_lo, nh, hl, split);
            for (int hh = lane; hh < nh; hh += 32) {
                md[2 * ((int64_t)slot * mdh + h_lo + hh)] = Mh[hh];
                md[2 * ((int64_t)slot * mdh + h_lo + hh) + 1] = Dh[hh];
            }
            __syncwarp();
        } else if constexpr (ASYNC) {
            reduce_edges_async<VEC, OP, COEF, U>(a, e0, e1, col, active, er_v, lane, acc, m, den);
        } else {
            Vec<VEC> xu;
            float *gout = nullptr;
            gatb_self<VEC, OP>(a, r, s, e0, col, active, xu, gout);
            reduce_edges<VEC, OP, COEF, U, G>(a, e0, e1, col, active, er_v, lane, acc, m, den, xu,
                                                 gout);
        }
        if (active && stores<G>(lane)) st_vec<VEC>(a.scratch + (int64_t)slot * a.ldp + col, acc);
        if constexpr (OP == OP_GAT)
            if (s == s0 && lane == 0) {
                md[2 * (int64_t)slot] = m;
                md[2 * (int64_t)slot + 1] = den;
            }
    }
    __threadfence();
    __syncwarp();
    int last = 0;
    if (lane == 0) last = (atomicAdd(ticket, 1) == nch - 1);
    last = __shfl_sync(FULL, last, 0);
    if (!last) return;
    __threadfence();
    float M = -INFINITY, D = 0.f;
    if constexpr (OP == OP_GAT) {
        for (int q = 0; q < nch; ++q) M = fmaxf(M, __ldcg(md + 2 * (int64_t)(off + q)));
        for (int q = 0; q < nch; ++q) {
            const float mq = __ldcg(md + 2 * (int64_t)(off + q));
            const float dq = __ldcg(md + 2 * (int64_t)(off + q) + 1);
            D = fmaf(dq, __expf(mq - M), D);
        }
    }
    for (int s = s0; s < s1; ++s) {
        const int col = strip_col<VEC, G>(a, s, lane);
        const bool active = in_strip<G>(a, lane, col);
        // OP_GATH: the lane's (up to two) heads and their merged softmax states
        int64_t mA = 0, mB = 0;
        int split = VEC;
        float MA = -INFINITY, DA = 0.f, MB = -INFINITY, DB = 0.f;
        if constexpr (OP == OP_GATH) {
            const int cc = active ? col : s * a.lps * VEC;
            mA = cc / a.fh;
            split = (int)((mA + 1) * a.fh - cc);
            mB = min(mA + (split < VEC ? 1 : 0), (int64_t)a.heads - 1);
            for (int q = 0; q < nch; ++q) {
                MA = fmaxf(MA, __ldcg(md + 2 * ((int64_t)(off + q) * mdh + mA)));
                MB = fmaxf(MB, __ldcg(md + 2 * ((int64_t)(off + q) * mdh + mB)));
            }
            for (int q = 0; q < nch; ++q) {
                const float *pa = md + 2 * ((int64_t)(off + q) * mdh + mA);
                const float *pb = md + 2 * ((int64_t)(off + q) * mdh + mB);
                DA = fmaf(__ldcg(pa + 1), __expf(__ldcg(pa) - MA), DA);
                DB = fmaf(__ldcg(pb + 1), __expf(__ldcg(pb) - MB), DB);
            }
        }
        Vec<VEC> acc;
#pragma unroll
        for (int c = 0; c < VEC; ++c) acc.v[c] = 0.f;
        if (active) {
            for (int q = 0; q < nch; ++q) {
                Vec<VEC> p = ld_vec_cg<VEC>(a.scratch + (int64_t)(off + q) * a.ldp + col);
                if constexpr (OP == OP_GATH) {
                    const float wA = __expf(__ldcg(md + 2 * ((int64_t)(off + q) * mdh + mA)) - MA);
                    const float wB = __expf(__ldcg(md + 2 * ((int64_t)(off + q) * mdh + mB)) - MB);
#pragma unroll
                    for (int c = 0; c < VEC; ++c) acc.v[c] = fmaf(c < split ? wA : wB, p.v[c], acc.v[c]);
                } else if constexpr (OP == OP_GAT) {
                    const float w = __expf(__ldcg(md + 2 * (int64_t)(off + q)) - M);
#pragma unroll
                    for (int c = 0; c < VEC; ++c) acc.v[c] = fmaf(w, p.v[c], acc.v[c]);
                } else {
#pragma unroll
                    for (int c = 0; c < VEC; ++c) acc.v[c] += p.v[c];
                }
            }
        }
        Vec<VEC> y;
        if constexpr (OP == OP_GATH) {
#pragma unroll
            for (int c = 0; c < VEC; ++c) y.v[c] = acc.v[c] / (c < split ? DA : DB);
            apply_layer_epilogue<VEC>(a, col, y);
        } else {
            y = epilogue<VEC, OP>(a, r, ee - eb, col, active, acc, D);
        }
        if (active && stores<G>(lane)) store_out<VEC>(a, r, col, y);
        if constexpr (OP != OP_GATH) project_row<VEC, G>(a, r, s, col, active, y, lane);
    }
    if (lane == 0) *ticket = 0;  // self-reset for the next launch
}

// Work item i: task-major (all strips of task i) or, in panel mode, strip
// s = i / n_tasks of task i % n_tasks, so that all warps sweep one L2-resident
// feature panel of X at a time.
template <int VEC, int OP, int COEF, int U, bool ASYNC, int G>
__device__ __forceinline__ void do_item(const AggArgs &a, int64_t i, int lane) {
    int64_t t = i;
    int s0 = 0, s1 = a.n_strips;
    if (a.panel) {
        s0 = (int)(i / a.n_tasks);
        t = i - (int64_t)s0 * a.n_tasks;
        s1 = s0 + 1;
    }
    const int2 tk = a.tasks[t];
    if (tk.y >= 0) do_unit<VEC, OP, COEF, U, ASYNC, G>(a, tk.x, tk.y, s0, s1, lane);
    else do_hub_chunk<VEC, OP, COEF, U, ASYNC, G>(a, tk.x, -tk.y - 1, s0, s1, lane);
}

// Resident CTAs per SM the kernel is compiled for (register budget).  The
// coefficient-free sums (GIN, SAGE, GCN NONE / RIGHT / pre-scaled BOTH) fit 64
// registers, so they run 32 warps per SM (measured: Reddit GIN 24.0 -> 21.8
// ms); ops with an edge coefficient (weighted, GAT) keep 85 registers (24
// warps), where fewer registers spill into the edge loop (measured slower;
// the alpha-mode GAT gather at 4 CTAs/SM: 26.9 -> 31.0 ms on Reddit).
constexpr int min_blocks(int op, int coef, bool async, int G = 1) {
    return async ? TLP_MINB_ASYNC
         : (TLP_SMEMC && G > 1 && coef != COEF_NONE && (op == OP_GCN || op == OP_GIN || op == OP_GATB))
               ? TLP_MINB_SMC
                 : ((op == OP_GIN || op == OP_SAGE || op == OP_GCN) && coef == COEF_NONE)
                       ? TLP_MINB_LIGHT : TLP_MINB;
}

template <int VEC, int OP, int COEF, int U, bool ASYNC, int G>
__device__ __forceinline__ void agg_body(const AggArgs &a) {
    const int lane = threadIdx.x & 31;
    const int64_t wid = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
    if (a.sched == S_HARDWARE) {  // one warp per item
        if (wid < a.n_items) do_item<VEC, OP, COEF, U, ASYNC, G>(a, wid, lane);
        if (a.n_dests > 0) __threadfence_system();
        return;
    }
    const int64_t W = ((int64_t)gridDim.x * blockDim.x) >> 5;
    const int64_t stride = W * a.step;
    int64_t t = wid * a.step;  // static first wave
    while (t < a.n_items) {
        unsigned long long v = 0;
        if (a.sched == S_DYNAMIC && lane == 0) v = atomicAdd(a.ctr, (unsigned long long)a.step);
        const int64_t tend = min(t + a.step, a.n_items);
        for (int64_t tt = t; tt < tend; ++tt) do_item<VEC, OP, COEF, U, ASYNC, G>(a, tt, lane);
        if (a.sched == S_DYNAMIC) t = stride + (int64_t)__shfl_sync(FULL, v, 0);
        else t += stride;
    }
    if (a.n_dests > 0) __threadfence_system();  // peer stores visible before the barrier
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

template <int VEC, int OP, int COEF, int U, bool ASYNC, int G>
__global__ void __launch_bounds__(TLP_MAXT, min_blocks(OP, COEF, ASYNC, G)) k_agg(const AggArgs a) {
    agg_body<VEC, OP, COEF, U, ASYNC, G>(a);
}

// ------------------------------------------------------------- dispatch --

constexpr int kU = TLP_U;  // source rows per gather group (2 groups in flight)

typedef void (*KernelFn)(const AggArgs);

template <int VEC, bool ASYNC, int G>
static KernelFn pick(int op, int coef) {
    if (op == OP_GCN) {
        switch (coef) {
            case COEF_NONE: return k_agg<VEC, OP_GCN, COEF_NONE, kU, ASYNC, G>;
            case COEF_COUT: return k_agg<VEC, OP_GCN, COEF_COUT, kU, ASYNC, G>;
            case COEF_W: return k_agg<VEC, OP_GCN, COEF_W, kU, ASYNC, G>;
            default: return k_agg<VEC, OP_GCN, COEF_W_COUT, kU, ASYNC, G>;
        }
    }
    if (op == OP_GIN)
        return coef & COEF_W ? k_agg<VEC, OP_GIN, COEF_W, kU, ASYNC, G>
                             : k_agg<VEC, OP_GIN, COEF_NONE, kU, ASYNC, G>;
    if (op == OP_SAGE) return k_agg<VEC, OP_SAGE, COEF_NONE, kU, ASYNC, G>;
    if constexpr (!ASYNC && G <= 2)
        if (op == OP_GATB) return k_agg<VEC, OP_GATB, COEF_W, kU, false, G>;
    return k_agg<VEC, OP_GAT, COEF_NONE, kU, ASYNC, G>;
}

// multi-head GAT: full-warp register path or cp.async ring
static KernelFn pick_mh(int vec, bool async_path) {
    if (async_path)
        return vec == 4 ? k_agg<4, OP_GATH, COEF_NONE, kU, true, 1>
                        : vec == 2 ? k_agg<2, OP_GATH, COEF_NONE, kU, true, 1>
                                   : k_agg<1, OP_GATH, COEF_NONE, kU, true, 1>;
    return vec == 4 ? k_agg<4, OP_GATH, COEF_NONE, kU, false, 1>
                    : vec == 2 ? k_agg<2, OP_GATH, COEF_NONE, kU, false, 1>
                               : k_agg<1, OP_GATH, COEF_NONE, kU, false, 1>;
}

// gather path: 0 register (full warp), 1 cp.async ring, 2 register with G
// lane groups (G = 2: PAIR half-warps; 4, 8: narrow rows; VEC = 4)
static KernelFn pick_kernel(int path, int vec, int op, int coef, int groups) {
    if (path == 2) {
        if (groups == 8) return pick<4, false, 8>(op, coef);
        if (groups == 4) return pick<4, false, 4>(op, coef);
        return pick<4, false, 2>(op, coef);
    }
    if (path == 1)
        return vec == 4 ? pick<4, true, 1>(op, coef) : vec == 2 ? pick<2, true, 1>(op, coef)
                                                               : pick<1, true, 1>(op, coef);
    return vec == 4 ? pick<4, false, 1>(op, coef) : vec == 2 ? pick<2, false, 1>(op, coef)
                                                             : pick<1, false, 1>(op, coef);
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
        // opt in to the device maximum once per kernel (never lowered afterwards)
        int dev = 0, mx = 0;
        cudaGetDevice(&dev);
        cudaDeviceGetAttribute(&mx, cudaDevAttrMaxSharedMemoryPerBlockOptin, dev);
        cudaFuncSetAttribute(fn, cudaFuncAttributeMaxDynamicSharedMemorySize, mx);
        cudaFuncSetAttribute(fn, cudaFuncAttributePreferredSharedMemoryCarveout, 100);
    }
    int nb = 0;
    if (cudaOccupancyMaxActiveBlocksPerMultiprocessor(&nb, fn, threads, smem) != cudaSuccess || nb < 1)
        nb = 1;
    if (n_cache < 64) cache[n_cache++] = {fn, threads, smem, nb};
    return nb;
}

static bool aligned(const void *p, size_t a) { return ((uintptr_t)p % a) == 0; }

// X'[u, f] = c_out[u] * X[u, f] for f < F (unweighted GCN BOTH); the pad
// columns of the last vector are zeroed (gathered, never stored to Y).
template <int VEC>
__global__ void k_prescale(const float *__restrict__ X, const float *__restrict__ c_out, int64_t n,
                           int64_t F, int64_t ldx, int64_t nvec, float *__restrict__ Xs) {
    const int64_t tot = n * nvec;
    for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < tot;
         i += (int64_t)gridDim.x * blockDim.x) {
        const int64_t u = i / nvec;
        const int64_t c = (i - u * nvec) * VEC;
        const float cu = __ldg(c_out + u);
        const float *src = X + u * ldx + c;
        float *dst = Xs + u * ldx + c;
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
        // the ragged last vector: columns [F, c + VEC) lie inside ldx (vec was
        // chosen from ldx % VEC) and are read by the gathers, so define them
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
    const char *e = getenv("TLP_HOT");
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
            const double budget = 0.6 * (double)g->l2_bytes;
            bool edge = 4.0 * (double)g->n_src * (double)r.ldx > budget &&
                        256.0 * (double)g->n_src > budget;
            if (const char *e = getenv("TLP_BOTH")) {
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
    if (r.op == OP_GAT) {
        const double budget = 0.6 * (double)g->l2_bytes;
        gat_alpha = vec == 4 && 4.0 * (double)g->n_src * (double)r.ldx > budget &&
                    256.0 * (double)g->n_src <= budget;
        if (const char *e = getenv("TLP_GAT")) {
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
            k_gat_alpha<<<(unsigned)pb, 256, 0, s>>>(g->rowptr, g->colidx, g->n_dst, r.el, r.er + g->row_offset,
                                                     r.slope, g->hub_row, g->n_hubs, g->H, g->galpha);
            g->launches += 1;
            cudaError_t e = cudaGetLastError();
            if (e != cudaSuccess) return cuda_error(e, "k_gat_alpha launch");
        }
        if (gat_alpha) {
            op = OP_GCN;  // Y[v] = sum_e alpha_e X[u_e]: unnormalised streamed-weight sum
            norm = TLP_NORM_NONE;
            coef = COEF_W;
            ew = g->galpha;
        }
    }
    // Unweighted GCN BOTH: one pass writes
    // X'[u] = c_out[u] X[u] (each term rounded once, as the oracle's product),
    // then every gather path sums X' rows with no per-edge coefficient, i.e.
    // the register budget and instruction count of GIN.  Same bits on every
    // path, schedule and partition (every path gathers the same X').
    const float *Xg = r.X;
    if (prescale) {
        const size_t need = sizeof(float) * ((size_t)g->n_src * (size_t)r.ldx) + 64;
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
        if (vec == 4)
            k_prescale<4><<<pb, 256, 0, s>>>(r.X, g->c_out, g->n_src, r.F, r.ldx, nvec, g->xs);
        else if (vec == 2)
            k_prescale<2><<<pb, 256, 0, s>>>(r.X, g->c_out, g->n_src, r.F, r.ldx, nvec, g->xs);
        else
            k_prescale<1><<<pb, 256, 0, s>>>(r.X, g->c_out, g->n_src, r.F, r.ldx, nvec, g->xs);
        g->launches += 1;
        cudaError_t e = cudaGetLastError();
        if (e != cudaSuccess) return cuda_error(e, "k_prescale launch");
        Xg = g->xs;
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
        if (const char *e = getenv("TLP_PANEL")) mode = atoi(e);
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
    if (const char *e = getenv("TLP_GROUPS")) {
        const int gq = atoi(e);
        if ((gq == 1 || gq == 2 || gq == 4 || gq == 8) && vec == 4 && lps == 32 && op != OP_GATH)
            groups = gq;
    }
    if (op == OP_GATB && groups > 2) groups = 2;  // the edge-dot trees exist for G <= 2
    const int strip_w = groups > 1 ? (32 / groups) * vec : lps * vec;
    const int n_strips = (int)((r.F + strip_w - 1) / strip_w);
    // Few tasks for the resident warps (small graphs): split every task into its
    // strips as separate work items too, so all SMs get work.
    if (!panel && !panel_off && n_strips > 1 && g->n_tasks < (int64_t)g->num_sms * 32 * 4) panel = 1;
    if (n_strips < 2) panel = 0;

    AggArgs a;
    a.rowptr = g->rowptr;
    a.colidx = g->colidx;
    a.ew = ew;
    a.c_out = cvec;
    a.X = Xg;
    a.Y = r.Y;
    a.el = r.el;
    a.er = r.er;
    a.tasks = g->tasks;
    a.hub_row = g->hub_row;
    a.hub_off = g->hub_off;
    a.ctr = reinterpret_cast<unsigned long long *>(g->ctr);
    a.done = g->ctr + 2;
    a.ldx = r.ldx;
    a.ldy = r.ldy;
    a.ldp = (r.F + 3) / 4 * 4;
    a.row_offset = g->row_offset;
    a.n_tasks = g->n_tasks;
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
    if (const char *e = getenv("TLP_GATHER")) {
        if (!strcmp(e, "reg")) async_path = false;
        else if (!strcmp(e, "async")) async_path = true;
    }
    if (groups > 1 || r.op == OP_GATB) async_path = false;  // OP_GATB: register path only
    const int path = groups > 1 ? 2 : (async_path ? 1 : 0);
    // hot-source L2 policy: cp.async path only (rows streamed from HBM)
    if (async_path && r.op != OP_GATH && r.op != OP_GATB) {
        unsigned thr = 0;
        tlp_status st = hot_threshold(g, panel ? (int64_t)strip_w : r.ldx, panel != 0, s, &thr);
        if (st != TLP_OK) return st;
        if (thr) {
            a.colidx = g->colidx_tag;
            a.hot_thr = thr;
            a.cold_first = 1;
            if (const char *e = getenv("TLP_HOT_COLD")) a.cold_first = atoi(e);
        }
    }
    KernelFn fn = (r.op == OP_GATH) ? pick_mh(vec, async_path) : pick_kernel(path, vec, op, coef, groups);
    const int wpc = g->warps_per_cta > 0 ? std::min(g->warps_per_cta, TLP_MAXT / 32) : 8;
    const int threads = 32 * wpc;
    size_t smem = async_path ? (size_t)wpc * TLP_DEPTH * 32 * vec * sizeof(float) : 0;
    if (r.op == OP_GATH)
        smem = (size_t)wpc * (kMhWarpFloats + (async_path ? TLP_DEPTH * 32 * vec : 0)) * sizeof(float);
    if (smem > 0 && sched == S_HARDWARE) occupancy_blocks(fn, threads, smem);  // sets attributes
    int64_t blocks;
    if (sched == S_HARDWARE) {
        blocks = (a.n_items + wpc - 1) / wpc;
    } else {
        int per_sm = occupancy_blocks(fn, threads, smem);
        if (const char *e = getenv("TLP_CTAS"))  // measurement: cap resident CTAs per SM
            if (atoi(e) > 0) per_sm = std::min(per_sm, atoi(e));
        blocks = (int64_t)per_sm * g->num_sms;
        int64_t need = (a.n_items + (int64_t)wpc * step - 1) / ((int64_t)wpc * step);
        if (blocks > need) blocks = need;  // tiny graphs: do not launch idle warps
    }
    if (blocks < 1) blocks = 1;
    if (blocks > 0x7fffffff) return set_error(TLP_ERR_UNSUPPORTED, "grid too large");
    fn<<<(unsigned)blocks, threads, smem, s>>>(a);
    g->launches += 1;
    cudaError_t e = cudaGetLastError();
    if (e != cudaSuccess) return cuda_error(e, "k_agg launch");
    if (want_proj) {
        const int pb = (int)std::min<int64_t>((g->n_dst + 255) / 256, (int64_t)g->num_sms * 8);
        k_proj_sum<<<pb, 256, 0, s>>>(g->proj, n_strips, g->n_dst, r.el_out, r.er_out);
        g->launches += 1;
        e = cudaGetLastError();
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

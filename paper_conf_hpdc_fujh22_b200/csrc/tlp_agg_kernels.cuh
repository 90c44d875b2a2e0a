// tlp_agg_kernels.cuh -- the aggregation kernel templates.
//
// Included by the kernel translation units tlp_k_*.cu (each instantiates one
// family of k_agg specialisations, so the library builds in parallel) and by
// tlp_agg.cu (dispatch, scalar passes and the C ABI).
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
#pragma once
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
enum Sched : int { S_DYNAMIC = 0, S_STATIC = 1, S_HARDWARE = 2, S_CLC = 4 };

constexpr unsigned FULL = 0xffffffffu;

// Compile-time tuning knobs: source rows per
// gather group (two groups in flight per warp) and the launch bounds.
#ifndef TLP_U
#define TLP_U 2        // register path: rows per gather group (2 groups in flight)
#endif
#ifndef TLP_MAXT
#define TLP_MAXT 256   // threads per CTA at most (8 warps)
#endif
#ifndef TLP_UNIT_SMEM
#define TLP_UNIT_SMEM 1  // unit loop state in shared memory (do_unit, coefficient-free sums)
#endif
#ifndef TLP_SCHED_SMEM
#define TLP_SCHED_SMEM 1  // scheduler loop state in shared memory (agg_body)
#endif
#ifndef TLP_MINB
#define TLP_MINB 3     // register path: 3 CTAs/SM -> <= 85 registers, 24 warps/SM
#endif
#ifndef TLP_MHB
#define TLP_MHB 4      // multi-head GAT: heads scored together per pass
#endif

#ifndef TLP_MINB_LIGHT
#define TLP_MINB_LIGHT 4  // register path, no edge coefficient (GIN, SAGE): <= 64 registers, 32 warps/SM
#endif
#ifndef TLP_MINB_MH_ASYNC
#define TLP_MINB_MH_ASYNC 2  // multi-head async path: per-head softmax state needs ~100 registers
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
    unsigned int *ctr;   // next work item (32-bit: n_items + W * step < 2^31)
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
    unsigned fh_magic;  // OP_GATH: ceil(2^32 / fh) when F < 2^16 and fh > 1 (x / fh = umulhi(x, magic)), else 0
    int mh_nh, mh_words;  // OP_GATH: heads one strip can touch; per-warp head-block floats
    // NEXT-2 fused all-gather: when n_dests > 0 every output row is stored to
    // dests[i] + (row_offset + r) * ldy for each destination (the Y_full of every
    // rank, mapped over NVLink) instead of to Y.
    float *const *dests;
    int n_dests;
    // NCCL symmetric window with NVLS multicast (NEXT-2): when mc is
    // set, one multimem store to mc + (row_offset + r) * ldy lands the row in
    // Y_full on every rank of the node (NVSwitch replicates it); dests is then
    // unused for data
    float *mc;
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
    // gather layout: X above is the array the edges
    // gather from -- the caller's X, or a 128-byte-aligned copy (padded rows, or
    // panel-major blocks of pw columns, block s at X + s * gps, row stride pw);
    // xown / ldown are the caller's X for the self rows of GIN / SAGE
    const float *xown;
    int64_t ldown;
    int64_t gps;
    int pw;
    // panel-mode item decode without a division: s = i / n_tasks =
    // umul64hi(i, tasks_magic) (tasks_magic = ceil(2^64 / n_tasks), exact for
    // i < 2^32; n_tasks == 1 is special-cased)
    unsigned long long tasks_magic;
    // short-row kernel (tlp_k_rows.cu): rows of in-degree > hub_H are skipped
    // when skip_hubs (their chunks run in the general kernel)
    int skip_hubs;
    int64_t hub_H;
    int stream_hint;  // L2 evict_first on the per-edge streams and Y stores (L2-panel mode)
    // debug visit counter (Alg. 1's exactly-once semantics):
    // visits[r] += 1 per finished (row, strip) store; NULL = off
    int32_t *visits;
};

// One finished (row, strip) of local row r (warp-uniform call).
__device__ __forceinline__ void count_visit(const AggArgs &a, int64_t r, int lane) {
    if (a.visits && lane == 0) atomicAdd(a.visits + r, 1);
}

constexpr unsigned kIdxMask = (1u << 27) - 1u;

// Per-thread L2 policies for tagged gathers (createpolicy once per task).
// mask: the index bits of a colidx entry (kIdxMask when the entries carry tags,
// else all 32 bits: untagged graphs may have 2^27 or more source vertices).
struct GPol {
    unsigned thr, mask;
    unsigned long long hot, cold;
};
__device__ __forceinline__ GPol make_gpol(const AggArgs &a) {
    GPol g;
    g.thr = a.hot_thr;
    g.mask = g.thr ? kIdxMask : 0xffffffffu;
    if (g.thr) {
        asm("createpolicy.fractional.L2::evict_last.b64 %0, 1.0;" : "=l"(g.hot));
        if (a.cold_first) asm("createpolicy.fractional.L2::evict_first.b64 %0, 1.0;" : "=l"(g.cold));
        else asm("createpolicy.fractional.L2::evict_normal.b64 %0, 1.0;" : "=l"(g.cold));
    } else {
        // untagged: every gather takes the default (evict_normal) policy, so the
        // copy is one instruction form whether or not the graph is tagged
        asm("createpolicy.fractional.L2::evict_normal.b64 %0, 1.0;" : "=l"(g.hot));
        g.cold = g.hot;
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

// pol != 0: the store carries that L2 cache policy (evict_first for Y in
// L2-panel mode)
template <int VEC>
__device__ __forceinline__ void st_vec(float *p, const Vec<VEC> &x, unsigned long long pol = 0ull) {
    if constexpr (VEC == 4) {
        if (pol)
            asm volatile("st.global.L1::no_allocate.L2::cache_hint.v4.f32 [%0], {%1, %2, %3, %4}, %5;"
                         ::"l"(p), "f"(x.v[0]), "f"(x.v[1]), "f"(x.v[2]), "f"(x.v[3]), "l"(pol) : "memory");
        else
            *reinterpret_cast<float4 *>(p) = make_float4(x.v[0], x.v[1], x.v[2], x.v[3]);
    } else if constexpr (VEC == 2) {
        *reinterpret_cast<float2 *>(p) = make_float2(x.v[0], x.v[1]);
    } else {
        *p = x.v[0];
    }
}

// Store only columns < F (the tail vector of a row may straddle F).
template <int VEC>
__device__ __forceinline__ void st_row(float *row, int col, int F, const Vec<VEC> &x,
                                       unsigned long long pol = 0ull) {
    if (col + VEC <= F) {
        st_vec<VEC>(row + col, x, pol);
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
// backward 36.3 -> 34.4 ms).  TLP_SMEMC 2 (default since round 2, session 3)
// keeps the chunk's coefficients in the owning lanes' registers instead and
// shuffles each step's coefficient at consume time (no shared-memory row, no
// per-chunk store and syncs): Reddit GAT 18.31 -> 17.92 ms per call against
// the half-warp-major shared row (interleaved A/B); 1 keeps the shared row.
#ifndef TLP_SMEMC
#define TLP_SMEMC 2
#endif
#ifndef TLP_MINB_SMC
#define TLP_MINB_SMC 4   // resident CTAs for the shared-memory-coefficient kernels
#endif
__device__ __forceinline__ float *chunk_coef_smem() {
    __shared__ __align__(16) float tlp_cw[TLP_MAXT / 32][32];
    return tlp_cw[threadIdx.x >> 5];
}
#ifndef TLP_PAIR_C2
#define TLP_PAIR_C2 1
#endif
// Slot of lane (edge) l's coefficient in the chunk row: half-warp-major for
// PAIR strips with two-step groups (consume_group reads a float2 per group).
template <int G, int U>
__device__ __forceinline__ int pair_coef_slot(int lane) {
    return (G == 2 && U == 2 && TLP_PAIR_C2) ? (lane & 1) * 16 + (lane >> 1) : lane;
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
template <int VEC, int U, bool HASC, int G, bool GUARD, int PHASE, bool SMC = false, bool SHC = false>
__device__ __forceinline__ void consume_group(int j, int n, int grp, const Vec<VEC> (&xv)[U],
                                              const float (&ck)[U], Vec<VEC> (&ac)[2],
                                              const float *cw = nullptr, float c_l = 0.f) {
    // PAIR (G = 2) with the coefficients in shared memory: the chunk row is
    // stored half-warp-major (edge p at (p & 1) * 16 + p / 2, see
    // pair_coef_slot), so a group's U = 2 steps read one aligned float2 -- one
    // shared-memory wavefront per two steps instead of one per step
    constexpr bool C2 = SMC && G == 2 && U == 2 && TLP_PAIR_C2;
    float2 c2 = make_float2(0.f, 0.f);
    if constexpr (C2) c2 = *reinterpret_cast<const float2 *>(cw + grp * 16 + j);
#pragma unroll
    for (int k = 0; k < U; ++k) {
        const int p = G * (j + k) + grp;
        const int ch = (G > 1) ? 0 : ((PHASE + k) & 1);
        // (the shuffle runs on every lane: lane groups past the chunk end take
        // a clamped index; their value is not used)
        float cvs = 0.f;
        if constexpr (HASC && SHC) cvs = __shfl_sync(FULL, c_l, GUARD ? min(p, n - 1) : p);
        if (!GUARD || p < n) {
            float cv = 0.f;
            if constexpr (C2) cv = k == 0 ? c2.x : c2.y;
            else if constexpr (HASC) cv = SHC ? cvs : (SMC ? cw[p] : ck[k]);
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

// ---- L2 stream hints --------------------------------
// In L2-panel mode the per-edge streams (colidx, edge coefficients such as
// GAT's alpha) and the Y stores are touched once per strip: loaded / stored
// with an L2 evict_first policy they do not evict the L2-resident panel of X
// that every edge gathers from (a.stream_hint; measured: Reddit GAT 19.4 ->
// 18.4 ms, GCN 16.7 -> 16.3; on HBM-streaming inputs it costs 2-3 %, so it is
// off there).  A cache policy only: no value changes.
__device__ __forceinline__ unsigned long long policy_evict_first() {
    unsigned long long p;
    asm("createpolicy.fractional.L2::evict_first.b64 %0, 1.0;" : "=l"(p));
    return p;
}
__device__ __forceinline__ int ld_stream(const int32_t *ptr, unsigned long long pol = 0ull) {
    if (!pol) return __ldg(ptr);
    int v;
    asm volatile("ld.global.nc.L1::no_allocate.L2::cache_hint.b32 %0, [%1], %2;"
                 : "=r"(v) : "l"(ptr), "l"(pol));
    return v;
}
__device__ __forceinline__ float ld_stream(const float *ptr, unsigned long long pol = 0ull) {
    if (!pol) return __ldg(ptr);
    float v;
    asm volatile("ld.global.nc.L1::no_allocate.L2::cache_hint.f32 %0, [%1], %2;"
                 : "=f"(v) : "l"(ptr), "l"(pol));
    return v;
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
__device__ __forceinline__ void reduce_edges(const AggArgs &a, int64_t e0, int64_t e1, int s,
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
    // lane-group coefficients: TLP_SMEMC 1 = chunk row in shared memory, read
    // at consume time; 2 = shuffled from the owning lane at consume time
    constexpr bool SHC = (TLP_SMEMC == 2) && HASC && (G > 1);
    constexpr bool SMC = (TLP_SMEMC == 1) && HASC && (G > 1);
    constexpr bool NOCK = SMC || SHC;  // no coefficient register per row in flight
    float *cw = SMC ? chunk_coef_smem() : nullptr;
    // lanes past F read column 0 of the strip (a valid address); their results
    // are never stored.  Panel-major gather layout: strip s is a block of pw
    // columns with row stride pw.
    const char *base;
    unsigned row_bytes;
    if (a.gps) {
        base = reinterpret_cast<const char *>(a.X + (int64_t)s * a.gps + (active ? col - s * a.pw : 0));
        row_bytes = (unsigned)a.pw * 4u;
    } else {
        base = reinterpret_cast<const char *>(a.X + (active ? col : 0));
        row_bytes = (unsigned)a.ldx * 4u;
    }
    const float *__restrict__ dep = (OP == OP_GAT) ? a.el : a.c_out;
    // 32-bit edge offsets relative to e0 (a row or hub chunk has < 2^31 edges)
    const int32_t *__restrict__ ci = a.colidx + e0;
    const float *__restrict__ wp = (COEF & COEF_W) ? a.ew + e0 : nullptr;
    const int len = (int)(e1 - e0);
    const int grp = lane / (32 / G);  // lane group (G > 1)
    const unsigned long long spol = a.stream_hint ? policy_evict_first() : 0ull;
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
            u0 = ld_stream(ci + lane, spol);
            if constexpr (COEF & COEF_W) w0 = ld_stream(wp + lane, spol);
        }
        if (lane < n1) {
            u1 = ld_stream(ci + 32 + lane, spol);
            if constexpr (COEF & COEF_W) w1 = ld_stream(wp + 32 + lane, spol);
        }
        if constexpr (DEP)
            if (lane < n0) d0 = __ldg(dep + u0);
        while (true) {
            // two chunks ahead: indices; one chunk ahead: index-dependent values
            const int n2 = min(32, len - off - 64);
            int u2 = 0;
            float w2 = 1.f;
            if (lane < n2) {
                u2 = ld_stream(ci + off + 64 + lane, spol);
                if constexpr (COEF & COEF_W) w2 = ld_stream(wp + off + 64 + lane, spol);
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
                cw[pair_coef_slot<G, U>(lane)] = c_l;
                __syncwarp();
            }
            Vec<VEC> xa[U], xb[U];
            float ca[U], cb[U];
            float g_l = 0.f;  // OP_GATB (partial chunk): this strip's dot of edge `lane`
            DotTree dt_;      // OP_GATB (full chunk): pending butterfly levels
            if (n0 == 32) {
                // full chunk: fully unrolled, compile-time shuffle lanes, no guards
                issue_group<VEC, U, HASC, G, false, NOCK>(base, row_bytes, 0, 32, grp, u0, c_l, xa, ca);
#pragma unroll
                for (int j = 0; j < STEPS; j += 2 * U) {
                    issue_group<VEC, U, HASC, G, false, NOCK>(base, row_bytes, j + U, 32, grp, u0, c_l, xb, cb);
                    consume_group<VEC, U, HASC, G, false, 0, SMC, SHC>(j, 32, grp, xa, ca, ac, cw, c_l);
                    if constexpr (GB) dot_tree<VEC, U, PAIR>(j, lane, xa, xu, dt_, gout + off);
                    if (j + 2 * U < STEPS)
                        issue_group<VEC, U, HASC, G, false, NOCK>(base, row_bytes, j + 2 * U, 32, grp, u0, c_l, xa, ca);
                    consume_group<VEC, U, HASC, G, false, U, SMC, SHC>(j + U, 32, grp, xb, cb, ac, cw, c_l);
                    if constexpr (GB) dot_tree<VEC, U, PAIR>(j + U, lane, xb, xu, dt_, gout + off);
                }
            } else {
                // partial chunk (n0 is warp-uniform: the guards never diverge)
                const int steps = (n0 + G - 1) / G;
                issue_group<VEC, U, HASC, G, true, NOCK>(base, row_bytes, 0, n0, grp, u0, c_l, xa, ca);
                for (int j = 0; j < steps; j += 2 * U) {
                    const bool more = j + U < steps;
                    if (more) issue_group<VEC, U, HASC, G, true, NOCK>(base, row_bytes, j + U, n0, grp, u0, c_l, xb, cb);
                    consume_group<VEC, U, HASC, G, true, 0, SMC, SHC>(j, n0, grp, xa, ca, ac, cw, c_l);
                    if constexpr (GB) dot_group<VEC, U, PAIR, true>(j, n0, lane, xa, xu, g_l);
                    if (j + 2 * U < steps)
                        issue_group<VEC, U, HASC, G, true, NOCK>(base, row_bytes, j + 2 * U, n0, grp, u0, c_l, xa, ca);
                    if (more) consume_group<VEC, U, HASC, G, true, U, SMC, SHC>(j + U, n0, grp, xb, cb, ac, cw, c_l);
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
#ifndef TLP_DEPTH_MH
#define TLP_DEPTH_MH 16  // multi-head GAT async ring depth (its scoring pauses the issue)
#endif
#ifndef TLP_MH_PAIRW
#define TLP_MH_PAIRW 1  // multi-head async pairs: weights read as float2 ahead of the wait
#endif
#ifndef TLP_ASYNC_PAIR
#define TLP_ASYNC_PAIR 1  // two edges per cp.async commit group (fewer waits per edge)
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
// cp.async of source row u (possibly tagged) with the hot/cold L2 policy into
// the shared-space address dst (a 32-bit offset: no generic-to-shared
// conversion per copy).
template <int VEC>
__device__ __forceinline__ void cp_async_x(unsigned dst, const char *base, unsigned u,
                                           unsigned row_bytes, const GPol &gp, bool pred) {
    const float *src = reinterpret_cast<const float *>(
        base + (unsigned long long)(u & gp.mask) * row_bytes);
    if constexpr (VEC == 4) {
        // two predicated forms with loop-invariant policies (no per-copy policy
        // select into a uniform register); ignore-src (!pred) zero-fills
        asm volatile("{\n\t.reg .pred pi, ph;\n\t"
                     "setp.eq.u32 pi, %2, 0;\n\t"
                     "setp.ge.u32 ph, %3, %4;\n\t"
                     "@ph cp.async.cg.shared.global.L2::cache_hint [%0], [%1], 16, pi, %5;\n\t"
                     "@!ph cp.async.cg.shared.global.L2::cache_hint [%0], [%1], 16, pi, %6;\n\t}\n"
                     ::"r"(dst), "l"(src), "r"((unsigned)pred), "r"(u), "r"(gp.thr), "l"(gp.hot), "l"(gp.cold));
    } else {
        const int bytes = pred ? 4 * VEC : 0;  // src-size 0 => zero fill, no global read
        if constexpr (VEC == 2)
            asm volatile("cp.async.ca.shared.global [%0], [%1], 8, %2;\n" ::"r"(dst), "l"(src), "r"(bytes));
        else
            asm volatile("cp.async.ca.shared.global [%0], [%1], 4, %2;\n" ::"r"(dst), "l"(src), "r"(bytes));
    }
}
// Lane l gets the index of edge l + K of the 64 held in (u0, u1): u0[l + K]
// while l + K < 32, else u1[l + K - 32] (two shuffles and a select per chunk
// instead of a select per issued edge).
template <int K>
__device__ __forceinline__ int ahead_index(int u0, int u1, int lane) {
    const int a0 = __shfl_sync(FULL, u0, (lane + K) & 31);
    const int a1 = __shfl_sync(FULL, u1, (lane + K) & 31);
    return lane + K < 32 ? a0 : a1;
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
        const unsigned ring_s = (unsigned)__cvta_generic_to_shared(ring);
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
            if (lane < n0) d0 = __ldg(dep + (u0 & gp.mask));
        if (len < D) {
            // short row (R-MAT / products have many): its rows go into ring
            // slots 0 .. len-1 under ONE commit group and one wait, instead of
            // the D-1 prologue groups and a wait per edge of the pipeline below
            // (same values, same order: bitwise the pipelined result)
            for (int k = 0; k < len; ++k) {
                const int uk = __shfl_sync(FULL, u0, k);
                cp_async_x<VEC>(ring_s + 4u * k * 32 * VEC, base, (unsigned)uk, row_bytes, gp, active);
            }
            cp_async_commit();
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
            cp_async_wait<0>();
            for (int j = 0; j < len; ++j) {
                const float cj = __shfl_sync(FULL, c_l, j);
                if (j & 1) acc_from_smem<VEC, HASC>(ring + j * 32 * VEC, cj, ao);
                else acc_from_smem<VEC, HASC>(ring + j * 32 * VEC, cj, ae);
            }
            __syncwarp();  // the ring is rewritten by the next row
#pragma unroll
            for (int c = 0; c < VEC; ++c) acc.v[c] = ae.v[c] + ao.v[c];
            return;
        }
#if TLP_ASYNC_PAIR
        // prologue: edges 0 .. D-3 in flight, two edges per commit group
        static_assert(D % 2 == 0, "paired async pipeline needs an even ring depth");
#pragma unroll
        for (int k = 0; k < D - 2; k += 2) {
            const int ua = __shfl_sync(FULL, k < 32 ? u0 : u1, k & 31);
            const int ub = __shfl_sync(FULL, k + 1 < 32 ? u0 : u1, (k + 1) & 31);
            cp_async_x<VEC>(ring_s + 4u * k * 32 * VEC, base, (unsigned)ua, row_bytes, gp, active && k < len);
            cp_async_x<VEC>(ring_s + 4u * (k + 1) * 32 * VEC, base, (unsigned)ub, row_bytes, gp, active && k + 1 < len);
            cp_async_commit();
        }
#else
        // prologue: edges 0 .. D-2 in flight
#pragma unroll
        for (int k = 0; k < D - 1; ++k) {
            const int uk = __shfl_sync(FULL, k < 32 ? u0 : u1, k & 31);
            cp_async_x<VEC>(ring_s + 4u * k * 32 * VEC, base, (unsigned)uk, row_bytes, gp, active && k < len);
            cp_async_commit();
        }
#endif
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
                if (lane < n1) d1 = __ldg(dep + (u1 & gp.mask));
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
#if TLP_ASYNC_PAIR
            // edges in pairs: one commit group and one wait per two edges; the
            // pair's first edge is at an even position (chunks start at even
            // offsets), so it feeds the even chain and the second the odd one
            // uq: lane l holds the index of edge l + D - 2 of this chunk (or of
            // the next chunk past its end), so the loop's two shuffles need no select
            const int uq = ahead_index<D - 2>(u0, u1, lane);
            for (int j = 0; j < n0; j += 2) {
                const int ja = j + D - 2, jb = j + D - 1;  // in this chunk or the next one
                const int ua = __shfl_sync(FULL, uq, j);
                const int ub = __shfl_sync(FULL, uq, j + 1);
                int wa = slot + D - 2;
                if (wa >= D) wa -= D;
                const int wb = wa + 1;  // slot and D are even
                cp_async_x<VEC>(ring_s + 4u * wa * 32 * VEC, base, (unsigned)ua, row_bytes, gp, active && (off + ja) < len);
                cp_async_x<VEC>(ring_s + 4u * wb * 32 * VEC, base, (unsigned)ub, row_bytes, gp, active && (off + jb) < len);
                cp_async_commit();
                cp_async_wait<(D - 2) / 2>();
                const float ca = __shfl_sync(FULL, c_l, j);
                const float cb = __shfl_sync(FULL, c_l, j + 1);  // lane j+1 mod 32: unused past n0
                acc_from_smem<VEC, HASC>(ring + slot * 32 * VEC, ca, ae);
                if (j + 1 < n0) acc_from_smem<VEC, HASC>(ring + (slot + 1) * 32 * VEC, cb, ao);
                slot += 2;
                if (slot == D) slot = 0;
            }
#else
            for (int j = 0; j < n0; ++j) {
                // issue edge j + D - 1 (in this chunk or the next one)
                const int jj = j + D - 1;
                const int ui = __shfl_sync(FULL, jj < 32 ? u0 : u1, jj & 31);
                const bool valid = (off + jj) < len;
                int ws = slot + D - 1;
                if (ws >= D) ws -= D;
                cp_async_x<VEC>(ring_s + 4u * ws * 32 * VEC, base, (unsigned)ui, row_bytes, gp, active && valid);
                cp_async_commit();
                cp_async_wait<D - 1>();
                const float cj = __shfl_sync(FULL, c_l, j);
                // chunks start at even offsets: the parity of j is the edge's parity
                if (j & 1) acc_from_smem<VEC, HASC>(ring + slot * 32 * VEC, cj, ao);
                else acc_from_smem<VEC, HASC>(ring + slot * 32 * VEC, cj, ae);
                if (++slot == D) slot = 0;
            }
#endif
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
// The per-warp head block (P, M, D, S) is sized at launch for the heads a
// strip can actually touch (a.mh_nh <= 33 for fh >= VEC; a.mh_words floats,
// a multiple of 4), so few heads leave room for more resident CTAs.
// x / fh for 0 <= x < F (a column index): one multiply-high by the host's
// ceil(2^32 / fh), exact for x * fh < 2^32 (F < 2^16), instead of a signed
// integer division sequence per row strip
__device__ __forceinline__ int mh_div(const AggArgs &a, int x) {
    return a.fh_magic ? (int)__umulhi((unsigned)x, a.fh_magic) : (int)((unsigned)x / (unsigned)a.fh);
}
__device__ __forceinline__ float *mh_warp_smem(const AggArgs &a) {
    extern __shared__ __align__(16) float tlp_smem[];
    return tlp_smem + (size_t)(threadIdx.x >> 5) * a.mh_words;
}

// The el values of one chunk's sources for the first TLP_MHB heads of a strip
// (lane j: source u_l of edge j), loaded ahead of the chunk's scoring so the
// dependent gather overlaps the previous chunk's row gathers.
__device__ __forceinline__ void mh_load_el(const AggArgs &a, unsigned u_l, int n0, int h_lo, int nh,
                                           int lane, float (&v)[TLP_MHB]) {
    const float *__restrict__ elu = a.el + (size_t)u_l * a.heads + h_lo;
#pragma unroll
    for (int k = 0; k < TLP_MHB; ++k) v[k] = (k < nh && lane < n0) ? __ldg(elu + k) : 0.f;
}

// Butterfly reduction of four values per lane at once (heads k = 0..3 of a
// block): after the first two exchange steps every lane carries one head,
// q = (lane >> 3) & 3, so the four reductions take 6 shuffles instead of 20.
// Each head's value is formed with the association of warp_sum / warp_max
// (own + partner at distances 16, 8, 4, 2, 1), so it is bitwise the
// one-value-at-a-time result; every lane of octet q holds head q's total.
template <bool MAX>
__device__ __forceinline__ float reduce4_transposed(const float (&v)[4], int lane) {
    auto op = [](float x, float y) { return MAX ? fmaxf(x, y) : x + y; };
    const bool hi = lane & 16;
    const float s0 = hi ? v[0] : v[2], s1 = hi ? v[1] : v[3];
    const float k0 = hi ? v[2] : v[0], k1 = hi ? v[3] : v[1];
    const float a0 = op(k0, __shfl_xor_sync(FULL, s0, 16));  // head 0 (2 on the upper half)
    const float a1 = op(k1, __shfl_xor_sync(FULL, s1, 16));  // head 1 (3)
    const bool b3 = lane & 8;
    float c = op(b3 ? a1 : a0, __shfl_xor_sync(FULL, b3 ? a0 : a1, 8));
#pragma unroll
    for (int o = 4; o > 0; o >>= 1) c = op(c, __shfl_xor_sync(FULL, c, o));
    return c;
}

// Scores, online-softmax update and weights of one 32-edge chunk for the heads
// [h_lo, h_lo+nh) of a strip (lane j holds edge j with source u_l), four heads
// per block: transposed max / sum reductions, and the running max, denominator
// and rescale of head q updated by lane 8q (all four in parallel); the first
// block's el / er values come in el0 / er0.
__device__ __forceinline__ void mh_chunk_scores(const AggArgs &a, unsigned u_l, int n0, int H, int h_lo,
                                                int nh, const float *__restrict__ erv,
                                                const float (&el0)[TLP_MHB], const float (&er0)[TLP_MHB],
                                                int lane, float *P, float *M, float *D, float *S) {
    static_assert(TLP_MHB == 4, "the transposed head reductions take four heads per block");
    constexpr int B = TLP_MHB;
    const float *__restrict__ elu = a.el + (size_t)u_l * H + h_lo;
    const int q = (lane >> 3) & 3;
    for (int hb = 0; hb < nh; hb += B) {
        float sv[B];
#pragma unroll
        for (int k = 0; k < B; ++k) {
            sv[k] = -INFINITY;
            if (hb + k < nh && lane < n0) {
                const float t = hb == 0 ? el0[k] + er0[k] : __ldg(elu + hb + k) + __ldg(erv + hb + k);
                sv[k] = t >= 0.f ? t : a.slope * t;  // LeakyReLU (R6)
            }
        }
        const bool mine = hb + q < nh;  // head q of this block exists
        const float mo = mine ? M[hb + q] : -INFINITY;
        const float mn = fmaxf(mo, reduce4_transposed<true>(sv, lane));
        float p[B];
#pragma unroll
        for (int k = 0; k < B; ++k) {
            const float mk = __shfl_sync(FULL, mn, 8 * k);
            p[k] = (lane < n0 && hb + k < nh) ? __expf(sv[k] - mk) : 0.f;
            if (hb + k < nh) P[(hb + k) * 32 + lane] = p[k];
        }
        const float sm = reduce4_transposed<false>(p, lane);
        if ((lane & 7) == 0 && mine) {
            const float scale = __expf(mo - mn);
            M[hb + q] = mn;
            D[hb + q] = fmaf(D[hb + q], scale, sm);
            S[hb + q] = scale;
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
    float *P = mh_warp_smem(a);
    float *M = P + a.mh_nh * 32;
    float *D = M + a.mh_nh;
    float *S = D + a.mh_nh;
    Mh = M;
    Dh = D;
    const int H = a.heads, fh = a.fh;
    const int c_lo = s * 32 * VEC;
    const int c_hi = min(a.F, c_lo + 32 * VEC) - 1;
    h_lo = mh_div(a, c_lo);
    nh = mh_div(a, c_hi) - h_lo + 1;
    const int cc = active ? col : c_lo;
    hl = mh_div(a, cc) - h_lo;
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
    float er0[TLP_MHB];
#pragma unroll
    for (int k = 0; k < TLP_MHB; ++k) er0[k] = k < nh ? __ldg(erv + k) : 0.f;
    const int len = (int)(e1 - e0);
    Vec<VEC> ac[2];
#pragma unroll
    for (int c = 0; c < VEC; ++c) ac[0].v[c] = ac[1].v[c] = 0.f;
    for (int off = 0; off < len; off += 32) {
        const int n0 = min(32, len - off);
        const int u_l = (lane < n0) ? __ldg(ci + off + lane) : 0;
        float el0[TLP_MHB];
        mh_load_el(a, (unsigned)u_l, n0, h_lo, nh, lane, el0);
        mh_chunk_scores(a, (unsigned)u_l, n0, H, h_lo, nh, erv, el0, er0, lane, P, M, D, S);
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
__device__ __forceinline__ float *mh_warp_smem_async(const AggArgs &a) {
    extern __shared__ __align__(16) float tlp_smem[];
    const int stride = a.mh_words + TLP_DEPTH_MH * 32 * VEC;
    return tlp_smem + (size_t)(threadIdx.x >> 5) * stride;
}

// The cp.async path mirrors reduce_edges_async: rows shorter than the ring go
// in under one commit group (their scores computed while the rows land), longer
// rows run the paired pipeline, two edges per commit group; the next chunk's
// indices and el values are loaded one chunk ahead; hot-source L2 policy on the
// gathers (tagged colidx).  Same values in the same order as the register path.
template <int VEC>
__device__ __forceinline__ void mh_consume(const float *src, float ca, float cb, int split, Vec<VEC> &ac) {
    if constexpr (VEC == 4) {
        const float4 x = *reinterpret_cast<const float4 *>(src);
        ac.v[0] = fmaf(0 < split ? ca : cb, x.x, ac.v[0]);
        ac.v[1] = fmaf(1 < split ? ca : cb, x.y, ac.v[1]);
        ac.v[2] = fmaf(2 < split ? ca : cb, x.z, ac.v[2]);
        ac.v[3] = fmaf(3 < split ? ca : cb, x.w, ac.v[3]);
    } else {
#pragma unroll
        for (int c = 0; c < VEC; ++c) ac.v[c] = fmaf(c < split ? ca : cb, src[c], ac.v[c]);
    }
}

template <int VEC>
__device__ __forceinline__ void reduce_edges_mh_async(const AggArgs &a, int64_t e0, int64_t e1,
                                                      int s, int col, bool active, int64_t rglob,
                                                      int lane, Vec<VEC> &acc, float *&Mh,
                                                      float *&Dh, int &h_lo, int &nh, int &hl,
                                                      int &split) {
    constexpr int DD = TLP_DEPTH_MH;
    static_assert(DD % 2 == 0, "paired async pipeline needs an even ring depth");
    float *P = mh_warp_smem_async<VEC>(a);
    float *M = P + a.mh_nh * 32;
    float *Dn = M + a.mh_nh;
    float *S = Dn + a.mh_nh;
    Mh = M;
    Dh = Dn;
    const int H = a.heads, fh = a.fh;
    const int c_lo = s * 32 * VEC;
    const int c_hi = min(a.F, c_lo + 32 * VEC) - 1;
    h_lo = mh_div(a, c_lo);
    nh = mh_div(a, c_hi) - h_lo + 1;
    const int cc = active ? col : c_lo;
    hl = mh_div(a, cc) - h_lo;
    split = (hl + h_lo + 1) * fh - cc;
    const int hl2 = min(hl + (split < VEC ? 1 : 0), nh - 1);
    for (int hh = lane; hh < nh; hh += 32) {
        M[hh] = -INFINITY;
        Dn[hh] = 0.f;
    }
    __syncwarp();
    const char *base = reinterpret_cast<const char *>(a.X + (active ? col : 0));
    const unsigned row_bytes = (unsigned)a.ldx * 4u;
    const GPol gp = make_gpol(a);
    const int32_t *__restrict__ ci = a.colidx + e0;
    const float *__restrict__ erv = a.er + rglob * H + h_lo;
    float er0[TLP_MHB];
#pragma unroll
    for (int k = 0; k < TLP_MHB; ++k) er0[k] = k < nh ? __ldg(erv + k) : 0.f;
    const int len = (int)(e1 - e0);
    const float *pa = P + hl * 32;
    const float *pb = P + hl2 * 32;
    Vec<VEC> ae, ao;
#pragma unroll
    for (int c = 0; c < VEC; ++c) ae.v[c] = ao.v[c] = 0.f;
    if (len > 0) {
        float *ring = P + a.mh_words + lane * VEC;
        const unsigned ring_s = (unsigned)__cvta_generic_to_shared(ring);
        int n0 = min(32, len), n1 = min(32, len - 32);
        int u0 = (lane < n0) ? ld_stream(ci + lane) : 0;
        int u1 = (lane < n1) ? ld_stream(ci + 32 + lane) : 0;
        float el0[TLP_MHB], el1[TLP_MHB];
        mh_load_el(a, (unsigned)u0 & gp.mask, n0, h_lo, nh, lane, el0);
        if (len < DD) {
            for (int k = 0; k < len; ++k) {
                const int uk = __shfl_sync(FULL, u0, k);
                cp_async_x<VEC>(ring_s + 4u * k * 32 * VEC, base, (unsigned)uk, row_bytes, gp, active);
            }
            cp_async_commit();
            // one chunk: the rescale of the (zero) chains is the identity
            mh_chunk_scores(a, (unsigned)u0 & gp.mask, n0, H, h_lo, nh, erv, el0, er0, lane, P, M, Dn, S);
#if TLP_MH_PAIRW
            cp_async_wait<0>();
            for (int j = 0; j < len; j += 2) {  // weights of edges j, j + 1 as two float2
                const float2 wA = *reinterpret_cast<const float2 *>(pa + j);
                const float2 wB = *reinterpret_cast<const float2 *>(pb + j);
                mh_consume<VEC>(ring + j * 32 * VEC, wA.x, wB.x, split, ae);
                if (j + 1 < len) mh_consume<VEC>(ring + (j + 1) * 32 * VEC, wA.y, wB.y, split, ao);
            }
#else
            cp_async_wait<0>();
            for (int j = 0; j < len; ++j) mh_consume<VEC>(ring + j * 32 * VEC, pa[j], pb[j], split, (j & 1) ? ao : ae);
#endif
            __syncwarp();  // P and the ring are rewritten by the next row
#pragma unroll
            for (int c = 0; c < VEC; ++c) acc.v[c] = ae.v[c] + ao.v[c];
            return;
        }
        // prologue: edges 0 .. DD-3 in flight, two edges per commit group
#pragma unroll
        for (int k = 0; k < DD - 2; k += 2) {
            const int ua = __shfl_sync(FULL, k < 32 ? u0 : u1, k & 31);
            const int ub = __shfl_sync(FULL, k + 1 < 32 ? u0 : u1, (k + 1) & 31);
            cp_async_x<VEC>(ring_s + 4u * k * 32 * VEC, base, (unsigned)ua, row_bytes, gp, active && k < len);
            cp_async_x<VEC>(ring_s + 4u * (k + 1) * 32 * VEC, base, (unsigned)ub, row_bytes, gp, active && k + 1 < len);
            cp_async_commit();
        }
        int slot = 0, off = 0;
        while (true) {
            const int n2 = min(32, len - off - 64);
            const int u2 = (lane < n2) ? ld_stream(ci + off + 64 + lane) : 0;
            if (n1 > 0) mh_load_el(a, (unsigned)u1 & gp.mask, n1, h_lo, nh, lane, el1);
            mh_chunk_scores(a, (unsigned)u0 & gp.mask, n0, H, h_lo, nh, erv, el0, er0, lane, P, M, Dn, S);
            const float sA = S[hl], sB = S[hl2];
#pragma unroll
            for (int c = 0; c < VEC; ++c) {
                const float sc = (c < split) ? sA : sB;
                ae.v[c] *= sc;
                ao.v[c] *= sc;
            }
            const int uq = ahead_index<DD - 2>(u0, u1, lane);
            for (int j = 0; j < n0; j += 2) {
                const int ja = j + DD - 2, jb = j + DD - 1;  // in this chunk or the next one
                const int ua = __shfl_sync(FULL, uq, j);
                const int ub = __shfl_sync(FULL, uq, j + 1);
                int wa = slot + DD - 2;
                if (wa >= DD) wa -= DD;
                const int wb = wa + 1;  // slot and DD are even
                cp_async_x<VEC>(ring_s + 4u * wa * 32 * VEC, base, (unsigned)ua, row_bytes, gp, active && (off + ja) < len);
                cp_async_x<VEC>(ring_s + 4u * wb * 32 * VEC, base, (unsigned)ub, row_bytes, gp, active && (off + jb) < len);
                cp_async_commit();
#if TLP_MH_PAIRW
                // the pair's weights as two float2 (j is even), read ahead of the wait
                const float2 wA = *reinterpret_cast<const float2 *>(pa + j);
                const float2 wB = *reinterpret_cast<const float2 *>(pb + j);
                cp_async_wait<(DD - 2) / 2>();
                mh_consume<VEC>(ring + slot * 32 * VEC, wA.x, wB.x, split, ae);
                if (j + 1 < n0) mh_consume<VEC>(ring + (slot + 1) * 32 * VEC, wA.y, wB.y, split, ao);
#else
                cp_async_wait<(DD - 2) / 2>();
                mh_consume<VEC>(ring + slot * 32 * VEC, pa[j], pb[j], split, ae);
                if (j + 1 < n0) mh_consume<VEC>(ring + (slot + 1) * 32 * VEC, pa[j + 1], pb[j + 1], split, ao);
#endif
                slot += 2;
                if (slot == DD) slot = 0;
            }
            __syncwarp();  // P, S are rewritten by the next chunk
            if (n1 <= 0) break;
            off += 32;
            n0 = n1; n1 = n2;
            u0 = u1; u1 = u2;
#pragma unroll
            for (int k = 0; k < TLP_MHB; ++k) el0[k] = el1[k];
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
__device__ __forceinline__ Vec<VEC> epilogue(const AggArgs &a, int64_t r, int deg, int col,
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
        if (active) xs = ld_vec<VEC>(a.xown + (a.row_offset + r) * a.ldown + col);
        else {
#pragma unroll
            for (int c = 0; c < VEC; ++c) xs.v[c] = 0.f;
        }
#pragma unroll
        for (int c = 0; c < VEC; ++c) y.v[c] = fmaf(a.eps1, xs.v[c], acc.v[c]);
    } else if constexpr (OP == OP_SAGE) {
        // mean over N(v) (+ v itself when sage_self): (X[v] + sum) / (deg + 1)
        const int cnt = deg + a.sage_self;
        const float inv = 1.0f / (float)(cnt > 1 ? cnt : 1);
        Vec<VEC> xs;
#pragma unroll
        for (int c = 0; c < VEC; ++c) xs.v[c] = 0.f;
        if (a.sage_self && active) xs = ld_vec<VEC>(a.xown + (a.row_offset + r) * a.ldown + col);
#pragma unroll
        for (int c = 0; c < VEC; ++c) y.v[c] = (xs.v[c] + acc.v[c]) * inv;
    } else {
        // GAT: Y = acc / den, as one reciprocal and VEC products (every
        // single-head path -- general, short-row, hub merge -- shares this)
        const float inv = deg > 0 ? 1.0f / den : 0.f;
#pragma unroll
        for (int c = 0; c < VEC; ++c) y.v[c] = acc.v[c] * inv;
    }
    apply_layer_epilogue<VEC>(a, col, y);
    return y;
}

// Store a finished output vector of local row r: to Y, or (fused all-gather)
// to the same global row of every destination buffer.
template <int VEC>
__device__ __forceinline__ void store_out(const AggArgs &a, int64_t r, int col, const Vec<VEC> &y) {
    if (a.mc) {
        float *p = a.mc + (a.row_offset + r) * a.ldy + col;
        if (VEC == 4 && col + 4 <= a.F) {
            asm volatile("multimem.st.relaxed.sys.global.v4.f32 [%0], {%1, %2, %3, %4};"
                         ::"l"(p), "f"(y.v[0]), "f"(y.v[VEC > 1 ? 1 : 0]), "f"(y.v[VEC > 2 ? 2 : 0]),
                           "f"(y.v[VEC > 3 ? 3 : 0]) : "memory");
        } else {
#pragma unroll
            for (int c = 0; c < VEC; ++c)
                if (col + c < a.F)
                    asm volatile("multimem.st.relaxed.sys.global.f32 [%0], %1;" ::"l"(p + c), "f"(y.v[c]) : "memory");
        }
        return;
    }
    if (a.n_dests == 0) {
        st_row<VEC>(a.Y + r * a.ldy, col, a.F, y, a.stream_hint ? policy_evict_first() : 0ull);
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

// Per-warp shared-memory copy of the row offsets (and GAT's er) of the rows a
// unit walks: they stay out of the registers while the edge loop runs (the
// edge loop is what the 64-register budget is for; round 2: row-level spills
// -> shared memory).
__device__ __forceinline__ int64_t *warp_rowptr_smem() {
    __shared__ int64_t tlp_rp[TLP_MAXT / 32][32];
    return tlp_rp[threadIdx.x >> 5];
}
__device__ __forceinline__ float *warp_er_smem() {
    __shared__ float tlp_er[TLP_MAXT / 32][32];
    return tlp_er[threadIdx.x >> 5];
}

// A regular work unit: whole rows [r0, r1), feature strips [s0, s1).
template <int VEC, int OP, int COEF, int U, bool ASYNC, int G>
__device__ __forceinline__ void do_unit(const AggArgs &a, int r0, int r1, int s0, int s1,
                                        int lane) {
    int64_t *rps = warp_rowptr_smem();
    float *ers = warp_er_smem();
#if TLP_UNIT_SMEM
    // the unit's loop state (row block, row, strip and their bounds) lives in
    // per-warp shared memory across the gather instead of spilled registers
    // (coefficient-free sums only: with a streamed edge coefficient the
    // reloads cost more spills than they save -- GAT alpha mode 18.40 -> 18.59
    // ms, L2 write sectors 188 M -> 312 M per launch)
    if constexpr (OP != OP_GATH && COEF == COEF_NONE) {
    __shared__ int tlp_unit_s[TLP_MAXT / 32][8];
    volatile int *ls = tlp_unit_s[threadIdx.x >> 5];
    __syncwarp();
    if (lane == 0) { ls[0] = r0; ls[1] = r1; ls[4] = s0; ls[5] = s1; }
    __syncwarp();
    for (; ls[0] < ls[1]; ) {
        const int rb = ls[0];
        const int nr = min(31, ls[1] - rb);
        __syncwarp();  // the previous block's offsets are consumed
        if (lane <= nr) rps[lane] = __ldg(a.rowptr + rb + lane);
        if constexpr (OP == OP_GAT)
            if (lane < nr) ers[lane] = __ldg(a.er + a.row_offset + rb + lane);
        if (lane == 0) { ls[2] = 0; ls[3] = nr; }
        __syncwarp();
        for (; ls[2] < ls[3]; ) {
            if (lane == 0) ls[6] = ls[4];
            __syncwarp();
            for (; ls[6] < ls[5]; ) {
                const int k = ls[2];
                const int s = ls[6];
                const int64_t e0 = rps[k];
                const int64_t e1 = rps[k + 1];
                const float er_v = (OP == OP_GAT) ? ers[k] : 0.f;
                const int r = ls[0] + k;
                const int col = strip_col<VEC, G>(a, s, lane);
                const bool active = in_strip<G>(a, lane, col);
                Vec<VEC> acc;
#pragma unroll
                for (int c = 0; c < VEC; ++c) acc.v[c] = 0.f;
                float m = -INFINITY, den = 0.f;
                if constexpr (ASYNC) {
                    reduce_edges_async<VEC, OP, COEF, U>(a, e0, e1, col, active, er_v, lane, acc, m, den);
                } else {
                    Vec<VEC> xu;
                    float *gout = nullptr;
                    gatb_self<VEC, OP>(a, r, s, e0, col, active, xu, gout);
                    reduce_edges<VEC, OP, COEF, U, G>(a, e0, e1, s, col, active, er_v, lane, acc, m, den,
                                                         xu, gout);
                }
                {
                    // reloaded after the gather
                    const int k2 = ls[2], s2 = ls[6];
                    const int r2 = ls[0] + k2;
                    const int deg = (int)(rps[k2 + 1] - rps[k2]);
                    const int col2 = strip_col<VEC, G>(a, s2, lane);
                    const bool active2 = in_strip<G>(a, lane, col2);
                    Vec<VEC> y = epilogue<VEC, OP>(a, r2, deg, col2, active2, acc, den);
                    if (active2 && stores<G>(lane)) store_out<VEC>(a, r2, col2, y);
                    count_visit(a, r2, lane);
                    project_row<VEC, G>(a, r2, s2, col2, active2, y, lane);
                }
                __syncwarp();
                if (lane == 0) ls[6] = ls[6] + 1;
                __syncwarp();
            }
            if (lane == 0) ls[2] = ls[2] + 1;
            __syncwarp();
        }
        if (lane == 0) ls[0] = ls[0] + 31;
        __syncwarp();
    }
    return;
    }
#endif
    for (int rb = r0; rb < r1; rb += 31) {
        const int nr = min(31, r1 - rb);
        // lanes fetch the row offsets of up to 31 rows at once (register caching
        // of the index boundary, Fig. 7a), parked in shared memory
        __syncwarp();  // the previous block's offsets are consumed
        if (lane <= nr) rps[lane] = __ldg(a.rowptr + rb + lane);
        if constexpr (OP == OP_GAT)
            if (lane < nr) ers[lane] = __ldg(a.er + a.row_offset + rb + lane);
        __syncwarp();
        for (int k = 0; k < nr; ++k) {
            const int64_t e0 = rps[k];
            const int64_t e1 = rps[k + 1];
            const float er_v = (OP == OP_GAT) ? ers[k] : 0.f;
            const int r = rb + k;
            const int deg = (int)(e1 - e0);
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
                    // one reciprocal per head and products, as the single-head epilogue
                    const float iA = (e1 > e0) ? 1.0f / dA : 0.f, iB = (e1 > e0) ? 1.0f / dB : 0.f;
                    Vec<VEC> y;
#pragma unroll
                    for (int c = 0; c < VEC; ++c) y.v[c] = acc.v[c] * (c < split ? iA : iB);
                    apply_layer_epilogue<VEC>(a, col, y);
                    if (active) store_out<VEC>(a, r, col, y);
                    count_visit(a, r, lane);
                    continue;
                } else if constexpr (ASYNC) {
                    reduce_edges_async<VEC, OP, COEF, U>(a, e0, e1, col, active, er_v, lane, acc, m, den);
                } else {
                    Vec<VEC> xu;
                    float *gout = nullptr;
                    gatb_self<VEC, OP>(a, r, s, e0, col, active, xu, gout);
                    reduce_edges<VEC, OP, COEF, U, G>(a, e0, e1, s, col, active, er_v, lane, acc, m, den,
                                                         xu, gout);
                }
                Vec<VEC> y = epilogue<VEC, OP>(a, r, deg, col, active, acc, den);
                if (active && stores<G>(lane)) store_out<VEC>(a, r, col, y);
                count_visit(a, r, lane);
                project_row<VEC, G>(a, r, s, col, active, y, lane);
            }
        }
    }
}

// One C-edge chunk of hub h (a8), feature strips [s0, s1).  The last chunk of
// the hub to finish these strips merges all its partials in chunk order and
// writes the row.  Tickets (and GAT (m, den) pairs) are kept per panel s0.
#ifndef TLP_HUB_INLINE
#define TLP_HUB_INLINE __forceinline__
#endif
template <int VEC, int OP, int COEF, int U, bool ASYNC, int G>
__device__ TLP_HUB_INLINE void do_hub_chunk(const AggArgs &a, int h, int j, int s0, int s1,
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
            reduce_edges<VEC, OP, COEF, U, G>(a, e0, e1, s, col, active, er_v, lane, acc, m, den, xu,
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
            const float iA = 1.0f / DA, iB = 1.0f / DB;
#pragma unroll
            for (int c = 0; c < VEC; ++c) y.v[c] = acc.v[c] * (c < split ? iA : iB);
            apply_layer_epilogue<VEC>(a, col, y);
        } else {
            y = epilogue<VEC, OP>(a, r, (int)(ee - eb), col, active, acc, D);
        }
        if (active && stores<G>(lane)) store_out<VEC>(a, r, col, y);
        count_visit(a, r, lane);
        if constexpr (OP != OP_GATH) project_row<VEC, G>(a, r, s, col, active, y, lane);
    }
    if (lane == 0) *ticket = 0;  // self-reset for the next launch
}

// Work item i: task-major (all strips of task i) or, in panel mode, strip
// s = i / n_tasks of task i % n_tasks, so that all warps sweep one L2-resident
// feature panel of X at a time.
template <int VEC, int OP, int COEF, int U, bool ASYNC, int G>
__device__ __forceinline__ void do_item(const AggArgs &a, int i, int lane) {
    // 32-bit item arithmetic (the host guarantees n_items + W * step < 2^31):
    // these values stay live across the whole task, so every register counts
    int t = i;
    int s0 = 0, s1 = a.n_strips;
    if (a.panel) {
        s0 = (a.n_tasks == 1) ? i : (int)__umul64hi((unsigned long long)(unsigned)i, a.tasks_magic);
        t = i - s0 * (int)a.n_tasks;
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
    return async ? (op == OP_GATH ? TLP_MINB_MH_ASYNC : TLP_MINB_ASYNC)
         : (TLP_SMEMC && G > 1 && coef != COEF_NONE && (op == OP_GCN || op == OP_GIN || op == OP_GATB))
               ? TLP_MINB_SMC
                 : ((op == OP_GIN || op == OP_SAGE || op == OP_GCN) && coef == COEF_NONE)
                       ? TLP_MINB_LIGHT : TLP_MINB;
}

// Cluster Launch Control work stealing (S_CLC, SURVEY 8(a) a4's Blackwell
// option): the grid has one CTA per block of wpc * step work items.  Each warp
// first does its own step items of its CTA's block; then, warp by warp (no CTA
// barrier), it asks the hardware to cancel a CTA that has not started yet
// (clusterlaunchcontrol.try_cancel, answered through the warp's own mbarrier)
// and does that CTA's whole block alone, until no launch is left to cancel.
// The request for the next block is issued before the current one is
// processed, so its latency hides behind the work.  No global atomics, no
// counter reset.  Register-path kernels only: with the cp.async kernels'
// cache-policy copies in the same kernel, ptxas 12.9 emits LDGSTS with an
// odd uniform-register descriptor (desc[UR1]: illegal instruction at run
// time), so the dispatcher runs those kernels with the atomic counter.
__device__ __forceinline__ void clc_request(unsigned res, unsigned bar) {
    asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], 16;\n" ::"r"(bar) : "memory");
    asm volatile("clusterlaunchcontrol.try_cancel.async.shared::cta.mbarrier::complete_tx::bytes.b128 [%0], [%1];\n"
                 ::"r"(res), "r"(bar) : "memory");
}
__device__ __forceinline__ void clc_wait(unsigned bar, unsigned phase) {
    asm volatile("{\n\t.reg .pred p;\n"
                 "CLC_WAIT:\n\t"
                 "mbarrier.try_wait.parity.shared::cta.b64 p, [%0], %1;\n\t"
                 "@!p bra CLC_WAIT;\n\t}\n" ::"r"(bar), "r"(phase) : "memory");
}
// the canceled CTA's x coordinate, or -1 when nothing was left to cancel
__device__ __forceinline__ int clc_result(unsigned res) {
    int bx, ok;
    asm volatile("{\n\t.reg .pred p;\n\t.reg .b128 r;\n\t"
                 "ld.shared.b128 r, [%2];\n\t"
                 "clusterlaunchcontrol.query_cancel.is_canceled.pred.b128 p, r;\n\t"
                 "selp.u32 %1, 1, 0, p;\n\t"
                 "@p clusterlaunchcontrol.query_cancel.get_first_ctaid::x.b32.b128 %0, r;\n\t}\n"
                 : "=r"(bx), "=r"(ok) : "r"(res) : "memory");
    return ok ? bx : -1;
}

template <int VEC, int OP, int COEF, int U, bool ASYNC, int G>
__device__ __forceinline__ void agg_clc(const AggArgs &a, int lane) {
    __shared__ __align__(16) uint4 clc_res[TLP_MAXT / 32];
    __shared__ __align__(8) unsigned long long clc_bar[TLP_MAXT / 32];
    const int wpc = (int)(blockDim.x >> 5), warp = (int)(threadIdx.x >> 5);
    const unsigned res = (unsigned)__cvta_generic_to_shared(&clc_res[warp]);
    const unsigned bar = (unsigned)__cvta_generic_to_shared(&clc_bar[warp]);
    if (lane == 0) {
        asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;\n" ::"r"(bar) : "memory");
        asm volatile("fence.mbarrier_init.release.cluster;\n" ::: "memory");
    }
    __syncwarp();
    const int n_items = (int)a.n_items;
    const int blk = wpc * a.step;  // work items of one CTA
    // own share of this CTA's block
    int t0 = (int)blockIdx.x * blk + warp * a.step, tend = min(t0 + a.step, n_items);
    unsigned phase = 0;
    while (true) {
        if (lane == 0) clc_request(res, bar);
        for (int tt = t0; tt < tend; ++tt) do_item<VEC, OP, COEF, U, ASYNC, G>(a, tt, lane);
        clc_wait(bar, phase);
        const int b = clc_result(res);
        asm volatile("fence.proxy.async.shared::cta;\n" ::: "memory");  // read before the next async write
        __syncwarp();
        if (b < 0) break;
        phase ^= 1u;
        t0 = b * blk;  // a canceled CTA's whole block
        tend = min(t0 + blk, n_items);
    }
}

template <int VEC, int OP, int COEF, int U, bool ASYNC, int G>
__device__ __forceinline__ void agg_body(const AggArgs &a) {
    const int lane = threadIdx.x & 31;
    const int wid = (int)((blockIdx.x * blockDim.x + threadIdx.x) >> 5);
    const int n_items = (int)a.n_items;
    if (a.sched == S_HARDWARE) {  // one warp per item
        if (wid < n_items) do_item<VEC, OP, COEF, U, ASYNC, G>(a, wid, lane);
        if (a.n_dests > 0) __threadfence_system();
        return;
    }
    if constexpr (!ASYNC) {
        if (a.sched == S_CLC) {
            agg_clc<VEC, OP, COEF, U, ASYNC, G>(a, lane);
            if (a.n_dests > 0) __threadfence_system();
            return;
        }
    }
    const int W = (int)((gridDim.x * blockDim.x) >> 5);
#if TLP_SCHED_SMEM
    // the batch start and item index live in per-warp shared memory across
    // the item (the register-bound kernels otherwise spill them to local
    // memory, whose write-backs reach L2 and DRAM once per item)
    __shared__ int tlp_sched_s[TLP_MAXT / 32][2];
    volatile int *ss = tlp_sched_s[threadIdx.x >> 5];
    if (lane == 0) ss[0] = wid * a.step;  // static first wave
    __syncwarp();
    while (ss[0] < n_items) {
        unsigned v = 0;
        if (a.sched == S_DYNAMIC && lane == 0) v = atomicAdd(a.ctr, (unsigned)a.step);
        __syncwarp();
        if (lane == 0) ss[1] = ss[0];
        __syncwarp();
        while (ss[1] < min(ss[0] + a.step, n_items)) {
            do_item<VEC, OP, COEF, U, ASYNC, G>(a, ss[1], lane);
            __syncwarp();
            if (lane == 0) ss[1] = ss[1] + 1;
            __syncwarp();
        }
        const int nt = (a.sched == S_DYNAMIC) ? W * a.step + (int)__shfl_sync(FULL, v, 0) : ss[0] + W * a.step;
        if (lane == 0) ss[0] = nt;
        __syncwarp();
    }
#else
    int t = wid * a.step;  // static first wave
    while (t < n_items) {
        // the next batch is claimed before this one is processed (its latency
        // hides behind the work); 32-bit counter
        unsigned v = 0;
        if (a.sched == S_DYNAMIC && lane == 0) v = atomicAdd(a.ctr, (unsigned)a.step);
        const int tend = min(t + a.step, n_items);
        for (int tt = t; tt < tend; ++tt) do_item<VEC, OP, COEF, U, ASYNC, G>(a, tt, lane);
        if (a.sched == S_DYNAMIC) t = W * a.step + (int)__shfl_sync(FULL, v, 0);
        else t += W * a.step;
    }
#endif
    if (a.n_dests > 0) __threadfence_system();  // peer stores visible before the barrier
    if (a.sched == S_DYNAMIC && lane == 0) {
        // last warp out resets the counter: no memset launch between calls
        __threadfence();
        if (atomicAdd(a.done, 1u) == (unsigned)(W - 1)) {
            *a.ctr = 0u;
            *a.done = 0u;
            __threadfence();
        }
    }
}

template <int VEC, int OP, int COEF, int U, bool ASYNC, int G>
__global__ void __launch_bounds__(TLP_MAXT, min_blocks(OP, COEF, ASYNC, G)) k_agg(const AggArgs a) {
    agg_body<VEC, OP, COEF, U, ASYNC, G>(a);
}

// ------------------------------------------------- kernel families --

constexpr int kU = TLP_U;  // source rows per gather group (2 groups in flight)

typedef void (*KernelFn)(const AggArgs);

template <int VEC, bool ASYNC, int G>
KernelFn pick(int op, int coef) {
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

// One function per kernel family, each defined in its own translation unit
// (tlp_k_*.cu).  op / coef select the specialisation inside the family.
KernelFn pick_reg_v4(int op, int coef);     // full warp, VEC 4
KernelFn pick_reg_v21(int vec, int op, int coef);  // full warp, VEC 2 / 1
KernelFn pick_async_v4(int op, int coef);   // cp.async ring, VEC 4
KernelFn pick_async_v21(int vec, int op, int coef);
KernelFn pick_g2(int op, int coef);         // PAIR half-warps (64-column strips)
KernelFn pick_g4(int op, int coef);         // 4 lane groups (narrow rows)
KernelFn pick_g8(int op, int coef);         // 8 lane groups
KernelFn pick_mh(int vec, bool async_path); // multi-head GAT
KernelFn pick_rows(int op, int coef, bool hint, int nsi, bool plain);  // short-row kernel (tlp_k_rows.cu), VEC 4

}  // namespace tlp

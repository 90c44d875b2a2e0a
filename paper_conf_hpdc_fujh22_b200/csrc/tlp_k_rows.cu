// tlp_k_rows.cu -- the short-row gather kernel.
//
// For graphs whose gathered rows are L2-resident and that have no hub rows
// (every in-degree <= H: Cora, Pubmed and other small graphs), the work is
// latency- and instruction-bound, not bandwidth-bound: ~4 edges per row, so
// the per-row overhead of the general persistent kernel (task decode, unit and
// strip loops, hub-merge machinery, its register spills) dominates.  This
// kernel maps one warp to one (row, 128-column strip) item, assigned
// round-robin over the resident warps (static: no counter atomics), with a
// register footprint that leaves 4 CTAs / 32 warps per SM, and the next
// item's row bounds prefetched while the current item gathers, so more independent
// rows are in flight per SM:
//   rowptr pair -> 32 indices per coalesced load (and the streamed edge
//   coefficient, or el[u] for GAT) -> up to U row gathers in flight per lane
//   -> epilogue -> one store.
// The reduction order is the canonical one of tlp_agg_kernels.cuh (two chains
// over the even / odd edge positions of the row, fmaf in CSR order, added
// even + odd; GAT: online softmax rescaled once per 32-edge chunk with the same
// butterfly reductions), so the output is bitwise identical to the general
// kernel's for the same coefficients.
#include "tlp_agg_kernels.cuh"

namespace tlp {

#ifndef TLP_ROWS_MINB
#define TLP_ROWS_MINB 4  // resident CTAs per SM (<= 64 registers)
#endif
#ifndef TLP_ROWS_MINB2
#define TLP_ROWS_MINB2 3  // two-strip items: resident CTAs per SM (<= 80 registers)
#endif
#ifndef TLP_ROWS_U
#define TLP_ROWS_U 8
#endif
constexpr int kRowsU = TLP_ROWS_U;  // row gathers in flight per lane

// The per-row factor of the epilogue (a9): GCN c_in, SAGE 1 / (deg + self),
// GAT 1 / den (0 for an empty row); GIN has none.  Written exactly as in
// epilogue() (tlp_agg_kernels.cuh), so every strip gets the same bits as the
// general kernel's.
template <int OP>
__device__ __forceinline__ float row_scale(const AggArgs &a, int deg, float den) {
    if constexpr (OP == OP_GCN) {
        float cin = 1.f;
        const float dc = (float)(deg > 1 ? deg : 1);
        if (a.norm == TLP_NORM_RIGHT) cin = 1.0f / dc;
        else if (a.norm == TLP_NORM_BOTH) cin = 1.0f / sqrtf(dc);
        return cin;
    } else if constexpr (OP == OP_SAGE) {
        const int cnt = deg + a.sage_self;
        return 1.0f / (float)(cnt > 1 ? cnt : 1);
    } else if constexpr (OP == OP_GAT) {
        return deg > 0 ? 1.0f / den : 0.f;
    }
    return 1.f;
}

// One chunk of <= 32 edges at offset `off` of the row starting at e0, step 1:
// lane j loads the chunk's j-th source index (and its streamed coefficient).
template <int COEF>
__device__ __forceinline__ void chunk_idx(const AggArgs &a, int64_t e0, int off, int n0, int lane, int &u_l,
                                          float &w0) {
    u_l = 0;
    w0 = 1.f;
    if (lane < n0) {
        u_l = __ldg(a.colidx + e0 + off + lane);
        if constexpr (COEF & COEF_W) w0 = __ldg(a.ew + e0 + off + lane);
    }
}

// Step 2: lane j's edge coefficient (GAT: the online-softmax weight after
// the chunk's rescale, which is applied to `ac`).
template <int OP, int COEF, bool HINT, int NSI>
__device__ __forceinline__ float chunk_weight(const AggArgs &a, int n0, float er_v, int lane, int u_l, float w0,
                                              float &m, float &den, Vec<4> (&ac)[NSI][2]) {
    constexpr bool DEP = (COEF & COEF_COUT) || (OP == OP_GAT);
    float d0 = 0.f, c_l = 1.f;
    if constexpr (DEP) {
        const float *dep = (OP == OP_GAT) ? a.el : a.c_out;
        if (lane < n0) d0 = __ldg(dep + (HINT ? (u_l & (int)kIdxMask) : u_l));
    }
    if constexpr (OP == OP_GAT) {
        float sc = -INFINITY;
        if (lane < n0) {
            const float t = d0 + er_v;
            sc = t >= 0.f ? t : a.slope * t;  // LeakyReLU (R6)
        }
        const float m_new = fmaxf(m, warp_max(sc));
        const float scale = __expf(m - m_new);
        c_l = (lane < n0) ? __expf(sc - m_new) : 0.f;
        den = fmaf(den, scale, warp_sum(c_l));
#pragma unroll
        for (int q = 0; q < NSI; ++q)
#pragma unroll
            for (int c = 0; c < 4; ++c) {
                ac[q][0].v[c] *= scale;
                ac[q][1].v[c] *= scale;
            }
        m = m_new;
    } else {
        if constexpr (COEF & COEF_COUT) c_l = d0;
        if constexpr (COEF & COEF_W) c_l *= w0;
    }
    return c_l;
}

// The gathers of one chunk (n0 edges, indices / coefficients in u_l / c_l)
// for this lane's columns: kRowsU rows in flight, two chains by position parity.
// Hot-source L2 policy (rows streamed from HBM): a tagged index
// carries its source's out-degree class in bits 27-31; hot sources are loaded
// L2::evict_last, the others evict_first.  A cache policy only.
template <bool HINT>
__device__ __forceinline__ Vec<4> ld_row_hint(const char *base, unsigned u, unsigned row_bytes, const GPol &gp) {
    if constexpr (!HINT) return ld_vec<4>(row_ptr(base, u, row_bytes));
    const float *p = reinterpret_cast<const float *>(base + (unsigned long long)(u & kIdxMask) * row_bytes);
    const unsigned long long pol = u >= gp.thr ? gp.hot : gp.cold;
    float4 t;
    asm volatile("ld.global.nc.L2::cache_hint.v4.f32 {%0, %1, %2, %3}, [%4], %5;"
                 : "=f"(t.x), "=f"(t.y), "=f"(t.z), "=f"(t.w) : "l"(p), "l"(pol));
    Vec<4> r;
    r.v[0] = t.x; r.v[1] = t.y; r.v[2] = t.z; r.v[3] = t.w;
    return r;
}

// One chunk: indices, then the first step's gathers, then the coefficients
// (the dependent c_out / el load and GAT's score reductions overlap the
// gathers in flight instead of preceding them), then the FMAs, then the
// remaining steps.  Gathers cover this lane's columns of NSI strips (strip q
// at byte offset soff[q] from base): kRowsU / NSI edges x NSI strips =
// kRowsU row vectors in flight per lane, two chains by edge position parity.
template <int OP, int COEF, bool HINT, int NSI>
__device__ __forceinline__ void chunk_run(const AggArgs &a, int64_t e0, int off, int n0, float er_v, int lane,
                                          const char *base, const unsigned (&soff)[NSI], unsigned row_bytes,
                                          float &m, float &den, Vec<4> (&ac)[NSI][2], const GPol &gp) {
    constexpr bool HASC = (COEF != COEF_NONE) || (OP == OP_GAT);
    constexpr int UE = kRowsU / NSI;  // edges per step
    // every step issues UE edges; past the chunk end the index is clamped (a
    // duplicate of a line already in flight).  Measured: guarding the surplus
    // loads with (uniform) branches instead was slower (Cora 22 -> 40 us,
    // Pubmed 53 -> 58 us: the loads no longer issue back to back); so was
    // requesting a long chunk's rows into L1 up front (prefetch.global.L1,
    // chunks > 16 edges: Cora 22.6 -> 26.7 us, Pubmed GAT 49.3 -> 51.3 us).
    int u_l;
    float w0;
    chunk_idx<COEF>(a, e0, off, n0, lane, u_l, w0);
    Vec<4> x[UE][NSI];
    auto issue = [&](int j) {
#pragma unroll
        for (int k = 0; k < UE; ++k) {
            const int p = min(j + k, n0 - 1);
            const unsigned u = (unsigned)__shfl_sync(FULL, u_l, p);
#pragma unroll
            for (int q = 0; q < NSI; ++q) x[k][q] = ld_row_hint<HINT>(base + soff[q], u, row_bytes, gp);
        }
    };
    issue(0);
    const float c_l = chunk_weight<OP, COEF, HINT, NSI>(a, n0, er_v, lane, u_l, w0, m, den, ac);
    for (int j = 0;;) {
#pragma unroll
        for (int k = 0; k < UE; ++k) {
            const float cv = HASC ? __shfl_sync(FULL, c_l, min(j + k, n0 - 1)) : 0.f;
            if (j + k < n0) {
                const int ch = (j + k) & 1;  // chunks start at multiples of 32: parity of the row position
#pragma unroll
                for (int q = 0; q < NSI; ++q)
#pragma unroll
                    for (int c = 0; c < 4; ++c) {
                        if constexpr (HASC) ac[q][ch].v[c] = fmaf(cv, x[k][q].v[c], ac[q][ch].v[c]);
                        else ac[q][ch].v[c] += x[k][q].v[c];
                    }
            }
        }
        j += UE;
        if (j >= n0) break;
        issue(j);
    }
}

// Work item i: row r = i / n_items_per_row and its NSI consecutive 128-column
// strips starting at strip NSI * (i mod n_items_per_row).  One index /
// coefficient load (and, for GAT, one score / softmax pass) per chunk serves
// the NSI strips.  Rows of in-degree > a.hub_H are skipped when a.skip_hubs
// (their hub chunks run in the general kernel).  (Whole-row items with the
// strips gathered one after another -- indices and GAT scores formed once
// for all strips -- measured slower on Pubmed GAT, 113.6 vs 65.7 us: fewer
// independent chains in flight per SM; NSI strips share each step's
// kRowsU loads instead.)
// PLAIN: the call has no layer epilogue, fused all-gather destinations,
// projections, stream hint or visit counter (one plain store per strip).
template <int OP, int COEF, bool HINT, int NSI, bool PLAIN>
__global__ void __launch_bounds__(256, NSI == 2 ? TLP_ROWS_MINB2 : TLP_ROWS_MINB) k_rows(const AggArgs a) {
    constexpr int VEC = 4;
    const int lane = threadIdx.x & 31;
    const int wid = (int)((blockIdx.x * blockDim.x + threadIdx.x) >> 5);
    const int W = (int)((gridDim.x * blockDim.x) >> 5);
    const int n_items = (int)a.n_items;
    const int ipr = (a.n_strips + NSI - 1) / NSI;  // items per row
    const unsigned row_bytes = (unsigned)a.ldx * 4u;
    auto row_of = [&](int i) {
        return (ipr == 1) ? i : (int)__umul64hi((unsigned long long)(unsigned)i, a.tasks_magic);
    };
    // the row bounds (and GAT's er) of the next item are loaded one item ahead:
    // lane 0 / 1 hold rowptr[r] / rowptr[r + 1], lane 2 er[r].  (Rows taken
    // longest first through a degree-sorted row order measured slower: Cora
    // 22.9 -> 25.2 us, Pubmed GAT 51.0 -> 54.0 us.)
    auto prefetch = [&](int i, int64_t &rp, float &erp) {
        if (i < n_items) {
            const int r = row_of(i);
            if (lane < 2) rp = __ldg(a.rowptr + r + lane);
            if constexpr (OP == OP_GAT)
                if (lane == 2) erp = __ldg(a.er + a.row_offset + r);
        }
    };
    int64_t rp_n = 0;
    float er_n = 0.f;
    prefetch(wid, rp_n, er_n);
    GPol gp;
    if constexpr (HINT) gp = make_gpol(a);
    for (int i = wid; i < n_items; i += W) {
        const int r = row_of(i);
        const int s0 = (i - r * ipr) * NSI;
        const int64_t e0 = __shfl_sync(FULL, rp_n, 0), e1 = __shfl_sync(FULL, rp_n, 1);
        const int len = (int)(e1 - e0);
        float er_v = 0.f;
        if constexpr (OP == OP_GAT) er_v = __shfl_sync(FULL, er_n, 2);
        prefetch(i + W, rp_n, er_n);
        if (a.skip_hubs && len > a.hub_H) continue;  // a hub row: done by its chunks
        const int col0 = s0 * 32 * VEC + lane * VEC;
        const bool active0 = col0 < a.F;
        const char *base = reinterpret_cast<const char *>(a.X + (active0 ? col0 : 0));
        // strip q's columns sit 128 floats to the right; a lane past F gathers
        // its strip-0 vector again (a line already in flight)
        unsigned soff[NSI];
#pragma unroll
        for (int q = 0; q < NSI; ++q) soff[q] = (active0 && col0 + q * 128 < a.F) ? (unsigned)q * 512u : 0u;
        Vec<VEC> ac[NSI][2];
#pragma unroll
        for (int q = 0; q < NSI; ++q)
#pragma unroll
            for (int c = 0; c < VEC; ++c) ac[q][0].v[c] = ac[q][1].v[c] = 0.f;
        float m = -INFINITY, den = 0.f;
        for (int off = 0; off < len; off += 32) {
            const int n0 = min(32, len - off);
            chunk_run<OP, COEF, HINT, NSI>(a, e0, off, n0, er_v, lane, base, soff, row_bytes, m, den, ac, gp);
        }
        // the row's scale, formed once for its NSI strips (the same fp32
        // expressions as the shared epilogue, so the same bits)
        const float sc = row_scale<OP>(a, len, den);
#pragma unroll
        for (int q = 0; q < NSI; ++q) {
            const int s = s0 + q;
            if (NSI > 1 && s >= a.n_strips) break;
            const int col = col0 + q * 128;
            const bool active = col < a.F;
            Vec<VEC> y;
#pragma unroll
            for (int c = 0; c < VEC; ++c) y.v[c] = ac[q][0].v[c] + ac[q][1].v[c];
            if constexpr (OP == OP_GIN || OP == OP_SAGE) {
                Vec<VEC> xs;
#pragma unroll
                for (int c = 0; c < VEC; ++c) xs.v[c] = 0.f;
                if (active && (OP == OP_GIN || a.sage_self))
                    xs = ld_vec<VEC>(a.xown + (a.row_offset + r) * a.ldown + col);
#pragma unroll
                for (int c = 0; c < VEC; ++c)
                    y.v[c] = (OP == OP_GIN) ? fmaf(a.eps1, xs.v[c], y.v[c]) : (xs.v[c] + y.v[c]) * sc;
            } else {
#pragma unroll
                for (int c = 0; c < VEC; ++c) y.v[c] *= sc;
            }
            if constexpr (PLAIN) {
                // no layer epilogue, fused all-gather, projection, stream
                // hint or visit counter on this call
                if (active) st_row<VEC>(a.Y + (int64_t)r * a.ldy, col, a.F, y);
            } else {
                apply_layer_epilogue<VEC>(a, col, y);
                if (active) store_out<VEC>(a, r, col, y);
                count_visit(a, r, lane);
                project_row<VEC, 1>(a, r, s, col, active, y, lane);
            }
        }
    }
    if (a.n_dests > 0) __threadfence_system();  // peer stores visible before the barrier
}

template <bool HINT, int NSI, bool PLAIN>
static KernelFn pick_rows_h(int op, int coef) {
    if (op == OP_GCN) {
        switch (coef) {
            case COEF_NONE: return k_rows<OP_GCN, COEF_NONE, HINT, NSI, PLAIN>;
            case COEF_COUT: return k_rows<OP_GCN, COEF_COUT, HINT, NSI, PLAIN>;
            case COEF_W: return k_rows<OP_GCN, COEF_W, HINT, NSI, PLAIN>;
            default: return k_rows<OP_GCN, COEF_W_COUT, HINT, NSI, PLAIN>;
        }
    }
    if (op == OP_GIN)
        return coef & COEF_W ? k_rows<OP_GIN, COEF_W, HINT, NSI, PLAIN> : k_rows<OP_GIN, COEF_NONE, HINT, NSI, PLAIN>;
    if (op == OP_SAGE) return k_rows<OP_SAGE, COEF_NONE, HINT, NSI, PLAIN>;
    if (op == OP_GAT) return k_rows<OP_GAT, COEF_NONE, HINT, NSI, PLAIN>;
    return nullptr;
}

template <bool PLAIN>
static KernelFn pick_rows_p(int op, int coef, bool hint, int nsi) {
    if (nsi == 2) return hint ? pick_rows_h<true, 2, PLAIN>(op, coef) : pick_rows_h<false, 2, PLAIN>(op, coef);
    return hint ? pick_rows_h<true, 1, PLAIN>(op, coef) : pick_rows_h<false, 1, PLAIN>(op, coef);
}

// hint: the gathers follow the hot-source L2 policy (tagged colidx);
// nsi: 128-column strips per work item (1 or 2; four measured slower: 2 CTAs
// per SM at ~100 registers, Cora 34.9 vs 23.5 us, Pubmed GAT 70.2 vs 48.1 us);
// plain: see k_rows
KernelFn pick_rows(int op, int coef, bool hint, int nsi, bool plain) {
    return plain ? pick_rows_p<true>(op, coef, hint, nsi) : pick_rows_p<false>(op, coef, hint, nsi);
}

}  // namespace tlp

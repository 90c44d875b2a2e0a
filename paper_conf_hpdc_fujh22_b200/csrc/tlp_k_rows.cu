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
#ifndef TLP_ROWS_U
#define TLP_ROWS_U 8
#endif
constexpr int kRowsU = TLP_ROWS_U;  // row gathers in flight per lane

// One chunk of <= 32 edges at offset `off` of the row starting at e0: lane j
// holds the chunk's j-th source index and its edge coefficient (GAT: the
// online-softmax weight after the chunk's rescale, applied to `ac`).
template <int OP, int COEF, bool HINT>
__device__ __forceinline__ void chunk_coef(const AggArgs &a, int64_t e0, int off, int n0, float er_v,
                                           int lane, int &u_l, float &c_l, float &m, float &den,
                                           Vec<4> (&ac)[2]) {
    constexpr bool DEP = (COEF & COEF_COUT) || (OP == OP_GAT);
    float d0 = 0.f, w0 = 1.f;
    u_l = 0;
    c_l = 1.f;
    if (lane < n0) {
        u_l = __ldg(a.colidx + e0 + off + lane);
        if constexpr (COEF & COEF_W) w0 = __ldg(a.ew + e0 + off + lane);
    }
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
        for (int c = 0; c < 4; ++c) {
            ac[0].v[c] *= scale;
            ac[1].v[c] *= scale;
        }
        m = m_new;
    } else {
        if constexpr (COEF & COEF_COUT) c_l = d0;
        if constexpr (COEF & COEF_W) c_l *= w0;
    }
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

template <int OP, int COEF, bool HINT>
__device__ __forceinline__ void chunk_gather(const char *base, unsigned row_bytes, int u_l, float c_l,
                                             int n0, Vec<4> (&ac)[2], const GPol &gp) {
    constexpr bool HASC = (COEF != COEF_NONE) || (OP == OP_GAT);
    // every lane group issues kRowsU gathers per step; past the chunk end the
    // index is clamped (a duplicate of a line already in flight).  Measured:
    // guarding the surplus loads with (uniform) branches instead was slower
    // (Cora 22 -> 40 us, Pubmed 53 -> 58 us: the loads no longer issue back
    // to back).
    for (int j = 0; j < n0; j += kRowsU) {
        Vec<4> x[kRowsU];
#pragma unroll
        for (int k = 0; k < kRowsU; ++k) {
            const int p = min(j + k, n0 - 1);
            const unsigned u = (unsigned)__shfl_sync(FULL, u_l, p);
            x[k] = ld_row_hint<HINT>(base, u, row_bytes, gp);
        }
#pragma unroll
        for (int k = 0; k < kRowsU; ++k) {
            const float cv = HASC ? __shfl_sync(FULL, c_l, min(j + k, n0 - 1)) : 0.f;
            if (j + k < n0) {
                const int ch = (j + k) & 1;  // chunks start at multiples of 32: parity of the row position
#pragma unroll
                for (int c = 0; c < 4; ++c) {
                    if constexpr (HASC) ac[ch].v[c] = fmaf(cv, x[k].v[c], ac[ch].v[c]);
                    else ac[ch].v[c] += x[k].v[c];
                }
            }
        }
    }
}

// Work item i: row r = i / n_strips and its 128-column strip s.  Rows of
// in-degree > a.hub_H are skipped when a.skip_hubs (their hub chunks run in the
// general kernel).  (Whole-row items -- indices and GAT scores formed once for
// all strips -- measured slower on Pubmed GAT, 113.6 vs 65.7 us: fewer
// independent chains in flight per SM.)
template <int OP, int COEF, bool HINT>
__global__ void __launch_bounds__(256, TLP_ROWS_MINB) k_rows(const AggArgs a) {
    constexpr int VEC = 4;
    const int lane = threadIdx.x & 31;
    const int wid = (int)((blockIdx.x * blockDim.x + threadIdx.x) >> 5);
    const int W = (int)((gridDim.x * blockDim.x) >> 5);
    const int n_items = (int)a.n_items;
    const unsigned row_bytes = (unsigned)a.ldx * 4u;
    auto row_of = [&](int i) {
        return (a.n_strips == 1) ? i : (int)__umul64hi((unsigned long long)(unsigned)i, a.tasks_magic);
    };
    // the row bounds (and GAT's er) of the next item are loaded one item ahead:
    // lane 0 / 1 hold rowptr[r] / rowptr[r + 1], lane 2 er[r]
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
        const int s = i - r * a.n_strips;
        const int64_t e0 = __shfl_sync(FULL, rp_n, 0), e1 = __shfl_sync(FULL, rp_n, 1);
        const int len = (int)(e1 - e0);
        float er_v = 0.f;
        if constexpr (OP == OP_GAT) er_v = __shfl_sync(FULL, er_n, 2);
        prefetch(i + W, rp_n, er_n);
        if (a.skip_hubs && len > a.hub_H) continue;  // a hub row: done by its chunks
        const int col = s * 32 * VEC + lane * VEC;
        const bool active = col < a.F;
        const char *base = reinterpret_cast<const char *>(a.X + (active ? col : 0));
        Vec<VEC> ac[2];
#pragma unroll
        for (int c = 0; c < VEC; ++c) ac[0].v[c] = ac[1].v[c] = 0.f;
        float m = -INFINITY, den = 0.f;
        for (int off = 0; off < len; off += 32) {
            const int n0 = min(32, len - off);
            int u_l;
            float c_l;
            chunk_coef<OP, COEF, HINT>(a, e0, off, n0, er_v, lane, u_l, c_l, m, den, ac);
            chunk_gather<OP, COEF, HINT>(base, row_bytes, u_l, c_l, n0, ac, gp);
        }
        Vec<VEC> acc;
#pragma unroll
        for (int c = 0; c < VEC; ++c) acc.v[c] = ac[0].v[c] + ac[1].v[c];
        Vec<VEC> y = epilogue<VEC, OP>(a, r, len, col, active, acc, den);
        if (active) store_out<VEC>(a, r, col, y);
        count_visit(a, r, lane);
        project_row<VEC, 1>(a, r, s, col, active, y, lane);
    }
    if (a.n_dests > 0) __threadfence_system();  // peer stores visible before the barrier
}

template <bool HINT>
static KernelFn pick_rows_h(int op, int coef) {
    if (op == OP_GCN) {
        switch (coef) {
            case COEF_NONE: return k_rows<OP_GCN, COEF_NONE, HINT>;
            case COEF_COUT: return k_rows<OP_GCN, COEF_COUT, HINT>;
            case COEF_W: return k_rows<OP_GCN, COEF_W, HINT>;
            default: return k_rows<OP_GCN, COEF_W_COUT, HINT>;
        }
    }
    if (op == OP_GIN) return coef & COEF_W ? k_rows<OP_GIN, COEF_W, HINT> : k_rows<OP_GIN, COEF_NONE, HINT>;
    if (op == OP_SAGE) return k_rows<OP_SAGE, COEF_NONE, HINT>;
    if (op == OP_GAT) return k_rows<OP_GAT, COEF_NONE, HINT>;
    return nullptr;
}

// hint: the gathers follow the hot-source L2 policy (tagged colidx)
KernelFn pick_rows(int op, int coef, bool hint) {
    return hint ? pick_rows_h<true>(op, coef) : pick_rows_h<false>(op, coef);
}

}  // namespace tlp

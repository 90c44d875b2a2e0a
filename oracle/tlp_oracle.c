/*
 * tlp_oracle.c -- plain, slow, single-threaded fp64 CPU oracle for the
 * TLPGNN graph-convolution (neighbor aggregation) hot path.
 *
 * TEST INFRASTRUCTURE ONLY.  Only tests/, __graft_entry__.smoke() and the
 * cpu_baseline / --impl reference legs of bench.py may load this library.
 * It shares no code, header, table or helper with the CUDA path
 * (paper_conf_hpdc_fujh22_b200/csrc), and it never includes include/tlp.h.
 *
 * Citations: "P:<line>" = /root/reference/PAPER.md line (HPDC'22 TLPGNN),
 * "c2 #k" = SURVEY.md section 8(c) reading k, restated in DESIGN.md.
 *
 * What it computes (Eq. 1: a_u = (+)_{v in N(u)} psi(h_u, e_vu, h_v)),
 * for a destination row v whose in-edges are e in [rowptr[v], rowptr[v+1]) with
 * source u = colidx[e] (the pull / in-edge CSR of Fig. 7):
 *
 *   GCN  ("weighted based on degree", "weighted sum";
 *         norm modes are c2 #1, #3, #4):
 *        Y[v,f] = c_in[v] * sum_e w_e * c_out[u] * X[u,f]
 *   GIN  (Xu et al. [51]; c2 #2, #5, #9):
 *        Y[v,f] = (1+eps) * X[row_offset+v, f] + sum_e w_e * X[u,f]
 *   GAT  (attention coefficient per edge, softmax over all the
 *         attentions of v, aggregate weighted by the softmax; Velickovic [43];
 *         c2 #5-#8): plain TWO-PASS softmax, deliberately not the online form.
 *
 * Alongside every output it returns the bound term A[v,f] = sum |terms| used by
 * the parity criterion |Y_gpu - Y| <= 1e-5 * A + 1e-6 (BASELINE.json north star).
 *
 * Arithmetic: every fp32 input is promoted to double; sums run in CSR order
 * in double; exp() is libm's.  No blocking, fusion or reordering.
 */
#include <math.h>
#include <stdint.h>
#include <stdlib.h>
#include <string.h>

#define ORACLE_NORM_NONE 0
#define ORACLE_NORM_RIGHT 1
#define ORACLE_NORM_BOTH 2

/* ---- structure ---------------------------------------------------------- */

/* In-degree of each destination row: number of entries in its CSR range
 * (c2 #3: unweighted edge counts; multi-edges and self-loops count). */
void oracle_in_degree(int64_t n_dst, const int64_t *rowptr, int32_t *in_deg)
{
    for (int64_t v = 0; v < n_dst; ++v)
        in_deg[v] = (int32_t)(rowptr[v + 1] - rowptr[v]);
}

/* Out-degree of each source vertex: number of edges whose source is u
 * (c2 #3).  A plain count over colidx. */
void oracle_out_degree(int64_t n_src, int64_t nnz, const int32_t *colidx,
                       int32_t *out_deg)
{
    for (int64_t u = 0; u < n_src; ++u)
        out_deg[u] = 0;
    for (int64_t e = 0; e < nnz; ++e)
        out_deg[colidx[e]] += 1;
}

/* CSR validity (SURVEY 8(b) create contract): rowptr[0]=0, monotone,
 * rowptr[n]=nnz, 0 <= colidx < n_src.  Returns 0 if valid, else 1. */
int oracle_csr_invalid(int64_t n_dst, int64_t n_src, int64_t nnz,
                       const int64_t *rowptr, const int32_t *colidx)
{
    if (rowptr[0] != 0)
        return 1;
    for (int64_t v = 0; v < n_dst; ++v)
        if (rowptr[v + 1] < rowptr[v])
            return 1;
    if (rowptr[n_dst] != nnz)
        return 1;
    for (int64_t e = 0; e < nnz; ++e)
        if (colidx[e] < 0 || (int64_t)colidx[e] >= n_src)
            return 1;
    return 0;
}

/* Destination-row partition balanced by edge count (north star: "destination-
 * row ranges balanced by edge count"; c1 "Partition", c2 #16):
 *   b_0 = 0, b_P = N,
 *   b_k = min{ r in [0,N] : rowptr[r] >= floor(k*E/P) }   for 0 < k < P.
 * Written as a linear scan (obviously correct, O(P*N)). */
void oracle_partition(int64_t n, const int64_t *rowptr, int parts,
                      int64_t *bounds)
{
    int64_t nnz = rowptr[n];
    bounds[0] = 0;
    for (int k = 1; k < parts; ++k) {
        int64_t target = ((int64_t)k * nnz) / parts; /* floor for nnz >= 0 */
        int64_t r = 0;
        while (r < n && rowptr[r] < target)
            ++r;
        bounds[k] = r;
    }
    bounds[parts] = n;
}

/* ---- aggregations -------------------------------------------------------- */

/* The destination rows to evaluate: rows[i] if rows != NULL, else i. */
static int64_t pick_row(const int64_t *rows, int64_t i)
{
    return rows ? rows[i] : i;
}

/* GCN (c1 row "GCN").  norm: 0 NONE (c_in=c_out=1), 1 RIGHT (c_in = 1/max(in_deg,1),
 * c_out = 1), 2 BOTH (c_in = 1/sqrt(max(in_deg,1)), c_out = 1/sqrt(max(out_deg,1))),
 * Kipf [26].  out_deg counts edges over the whole CSR given (c2 #3).
 * ew may be NULL (w_e = 1); weights multiply, degrees stay unweighted (c2 #4).
 * Outputs Y[i*F + f] and (if A != NULL) A[i*F + f] for i < n_rows.
 * Returns 0, or -1 on bad arguments / allocation failure. */
int oracle_gcn(int64_t n_dst, int64_t n_src, const int64_t *rowptr,
               const int32_t *colidx, const float *ew, const float *X,
               int64_t F, int64_t ldx, int norm, int64_t n_rows,
               const int64_t *rows, double *Y, double *A)
{
    if (norm < 0 || norm > 2 || F < 0 || ldx < F)
        return -1;
    int64_t nnz = rowptr[n_dst];
    int32_t *out_deg = NULL;
    if (norm == ORACLE_NORM_BOTH) {
        out_deg = (int32_t *)malloc(sizeof(int32_t) * (size_t)(n_src > 0 ? n_src : 1));
        if (!out_deg)
            return -1;
        oracle_out_degree(n_src, nnz, colidx, out_deg);
    }
    for (int64_t i = 0; i < n_rows; ++i) {
        int64_t v = pick_row(rows, i);
        int64_t deg = rowptr[v + 1] - rowptr[v];
        double dclamp = (double)(deg > 1 ? deg : 1);
        double c_in = 1.0;
        if (norm == ORACLE_NORM_RIGHT)
            c_in = 1.0 / dclamp;
        else if (norm == ORACLE_NORM_BOTH)
            c_in = 1.0 / sqrt(dclamp);
        for (int64_t f = 0; f < F; ++f) {
            double s = 0.0, a = 0.0;
            for (int64_t e = rowptr[v]; e < rowptr[v + 1]; ++e) {
                int64_t u = colidx[e];
                double w = ew ? (double)ew[e] : 1.0;
                double c_out = 1.0;
                if (norm == ORACLE_NORM_BOTH) {
                    int32_t od = out_deg[u];
                    c_out = 1.0 / sqrt((double)(od > 1 ? od : 1));
                }
                double term = w * c_out * (double)X[u * ldx + f];
                s += term;
                a += fabs(term);
            }
            Y[i * F + f] = c_in * s;
            if (A)
                A[i * F + f] = c_in * a;
        }
    }
    free(out_deg);
    return 0;
}

/* GIN (c1 row "GIN"): Y[v,f] = (1+eps) X[row_offset+v, f] + sum_e w_e X[u,f].
 * The self row of destination v is X[row_offset + v] (row_offset = 0 for a
 * whole graph, b_k for a row slice).  Requires row_offset + n_dst <= n_src. */
int oracle_gin(int64_t n_dst, int64_t n_src, const int64_t *rowptr,
               const int32_t *colidx, const float *ew, const float *X,
               int64_t F, int64_t ldx, double eps, int64_t row_offset,
               int64_t n_rows, const int64_t *rows, double *Y, double *A)
{
    if (F < 0 || ldx < F || row_offset < 0 || row_offset + n_dst > n_src)
        return -1;
    double self_w = 1.0 + eps;
    for (int64_t i = 0; i < n_rows; ++i) {
        int64_t v = pick_row(rows, i);
        for (int64_t f = 0; f < F; ++f) {
            double self = self_w * (double)X[(row_offset + v) * ldx + f];
            double s = self, a = fabs(self);
            for (int64_t e = rowptr[v]; e < rowptr[v + 1]; ++e) {
                int64_t u = colidx[e];
                double w = ew ? (double)ew[e] : 1.0;
                double term = w * (double)X[u * ldx + f];
                s += term;
                a += fabs(term);
            }
            Y[i * F + f] = s;
            if (A)
                A[i * F + f] = a;
        }
    }
    return 0;
}

/* LeakyReLU, c2 #6: x >= 0 ? x : slope*x. */
static double leaky_relu(double x, double slope)
{
    return x >= 0.0 ? x : slope * x;
}

/* GAT, single head (c1 row "GAT").  For destination v with
 * in-degree d > 0:
 *   t_e = el[u] + er[row_offset+v];  s_e = LeakyReLU(t_e, slope)
 *   m = max_e s_e;  z = sum_e exp(s_e - m);  alpha_e = exp(s_e - m) / z
 *   Y[v,f] = sum_e alpha_e X[u,f];  A[v,f] = sum_e alpha_e |X[u,f]|
 * d = 0 gives Y = A = 0 (c2 #8).  Edge weights are not an input (c2 #5).
 * If alpha_sum != NULL, alpha_sum[i] = sum_e alpha_e (pin P5), 0 for d = 0. */
int oracle_gat(int64_t n_dst, int64_t n_src, const int64_t *rowptr,
               const int32_t *colidx, const float *X, int64_t F, int64_t ldx,
               const float *el, const float *er, double slope,
               int64_t row_offset, int64_t n_rows, const int64_t *rows,
               double *Y, double *A, double *alpha_sum)
{
    (void)n_src;
    if (F < 0 || ldx < F || row_offset < 0)
        return -1;
    for (int64_t i = 0; i < n_rows; ++i) {
        int64_t v = pick_row(rows, i);
        int64_t e0 = rowptr[v], e1 = rowptr[v + 1];
        int64_t d = e1 - e0;
        if (d == 0) {
            for (int64_t f = 0; f < F; ++f) {
                Y[i * F + f] = 0.0;
                if (A)
                    A[i * F + f] = 0.0;
            }
            if (alpha_sum)
                alpha_sum[i] = 0.0;
            continue;
        }
        double *alpha = (double *)malloc(sizeof(double) * (size_t)d);
        if (!alpha)
            return -1;
        /* pass 1: scores and their maximum */
        double er_v = (double)er[row_offset + v];
        double m = -INFINITY;
        for (int64_t e = e0; e < e1; ++e) {
            double s = leaky_relu((double)el[colidx[e]] + er_v, slope);
            alpha[e - e0] = s;
            if (s > m)
                m = s;
        }
        /* pass 2: normaliser, then the softmax weights */
        double z = 0.0;
        for (int64_t k = 0; k < d; ++k)
            z += exp(alpha[k] - m);
        double asum = 0.0;
        for (int64_t k = 0; k < d; ++k) {
            alpha[k] = exp(alpha[k] - m) / z;
            asum += alpha[k];
        }
        if (alpha_sum)
            alpha_sum[i] = asum;
        /* aggregation weighted by the softmax */
        for (int64_t f = 0; f < F; ++f) {
            double s = 0.0, a = 0.0;
            for (int64_t e = e0; e < e1; ++e) {
                double x = (double)X[(int64_t)colidx[e] * ldx + f];
                s += alpha[e - e0] * x;
                a += alpha[e - e0] * fabs(x);
            }
            Y[i * F + f] = s;
            if (A)
                A[i * F + f] = a;
        }
        free(alpha);
    }
    return 0;
}

/* ---- NEXT-1: GraphSage mean, multi-head GAT ------------------ */

/* GraphSage mean aggregator (Hamilton et al. [15]):
 *   include_self = 0:  Y[v,f] = (1/max(d,1)) * sum_e X[u,f]            (mean of N(v))
 *   include_self = 1:  Y[v,f] = (X[row_offset+v,f] + sum_e X[u,f]) / (d+1)
 *                      (the "GCN" aggregator variant of [15]: mean over N(v) + v)
 * Edge weights are not an input (the mean is unweighted).  A = sum |terms| / count. */
int oracle_sage(int64_t n_dst, int64_t n_src, const int64_t *rowptr,
                const int32_t *colidx, const float *X, int64_t F, int64_t ldx,
                int include_self, int64_t row_offset, int64_t n_rows,
                const int64_t *rows, double *Y, double *A)
{
    if (F < 0 || ldx < F || row_offset < 0 ||
        (include_self && row_offset + n_dst > n_src))
        return -1;
    for (int64_t i = 0; i < n_rows; ++i) {
        int64_t v = pick_row(rows, i);
        int64_t d = rowptr[v + 1] - rowptr[v];
        int64_t cnt = d + (include_self ? 1 : 0);
        double inv = 1.0 / (double)(cnt > 1 ? cnt : 1);
        for (int64_t f = 0; f < F; ++f) {
            double s = 0.0, a = 0.0;
            if (include_self) {
                double x = (double)X[(row_offset + v) * ldx + f];
                s += x;
                a += fabs(x);
            }
            for (int64_t e = rowptr[v]; e < rowptr[v + 1]; ++e) {
                double x = (double)X[(int64_t)colidx[e] * ldx + f];
                s += x;
                a += fabs(x);
            }
            Y[i * F + f] = inv * s;
            if (A)
                A[i * F + f] = inv * a;
        }
    }
    return 0;
}

/* Multi-head GAT (Velickovic [43]): H heads, head h owns the
 * feature columns [h*Fh, (h+1)*Fh) of X and Y (F = H*Fh), with its own scores
 *   s_e,h = LeakyReLU(el[u*H + h] + er[(row_offset+v)*H + h], slope)
 * and its own softmax over the in-edges of v.  Each head is exactly the
 * single-head oracle_gat on its column block (computed here the same way). */
int oracle_gat_mh(int64_t n_dst, int64_t n_src, const int64_t *rowptr,
                  const int32_t *colidx, const float *X, int64_t H, int64_t Fh,
                  int64_t ldx, const float *el, const float *er, double slope,
                  int64_t row_offset, int64_t n_rows, const int64_t *rows,
                  double *Y, double *A)
{
    if (H < 1 || Fh < 0 || ldx < H * Fh || row_offset < 0)
        return -1;
    int64_t F = H * Fh;
    for (int64_t i = 0; i < n_rows; ++i) {
        int64_t v = pick_row(rows, i);
        int64_t e0 = rowptr[v], e1 = rowptr[v + 1];
        int64_t d = e1 - e0;
        double *alpha = (double *)malloc(sizeof(double) * (size_t)(d > 0 ? d : 1));
        if (!alpha)
            return -1;
        for (int64_t h = 0; h < H; ++h) {
            if (d > 0) {
                double er_v = (double)er[(row_offset + v) * H + h];
                double m = -INFINITY;
                for (int64_t e = e0; e < e1; ++e) {
                    double s = leaky_relu((double)el[(int64_t)colidx[e] * H + h] + er_v, slope);
                    alpha[e - e0] = s;
                    if (s > m)
                        m = s;
                }
                double z = 0.0;
                for (int64_t k = 0; k < d; ++k)
                    z += exp(alpha[k] - m);
                for (int64_t k = 0; k < d; ++k)
                    alpha[k] = exp(alpha[k] - m) / z;
            }
            for (int64_t f = h * Fh; f < (h + 1) * Fh; ++f) {
                double s = 0.0, a = 0.0;
                for (int64_t e = e0; e < e1; ++e) {
                    double x = (double)X[(int64_t)colidx[e] * ldx + f];
                    s += alpha[e - e0] * x;
                    a += alpha[e - e0] * fabs(x);
                }
                Y[i * F + f] = s;
                if (A)
                    A[i * F + f] = a;
            }
        }
        free(alpha);
    }
    return 0;
}

/* ---- NEXT-3: the layer epilogue of Eq. 2 ---------------------- */

/* h' = sigma(a + b) (Eq. 2; bias and activation of the layer).
 * act: 0 identity, 1 ReLU max(x,0), 2 LeakyReLU (x >= 0 ? x : p*x),
 *      3 ELU (x > 0 ? x : p*(exp(x)-1)).  bias may be NULL.  In place on Y
 * [n_rows x F]; the bound term A gains the bias as one more term (|b|), and the
 * activations used here are 1-Lipschitz for 0 <= p <= 1, so A bounds them too. */
int oracle_epilogue(int64_t n_rows, int64_t F, double *Y, double *A,
                    const float *bias, int act, double p)
{
    if (act < 0 || act > 3 || F < 0)
        return -1;
    for (int64_t i = 0; i < n_rows; ++i) {
        for (int64_t f = 0; f < F; ++f) {
            double x = Y[i * F + f];
            if (bias) {
                x += (double)bias[f];
                if (A)
                    A[i * F + f] += fabs((double)bias[f]);
            }
            if (act == 1)
                x = x > 0.0 ? x : 0.0;
            else if (act == 2)
                x = x >= 0.0 ? x : p * x;
            else if (act == 3)
                x = x > 0.0 ? x : p * (exp(x) - 1.0);
            Y[i * F + f] = x;
        }
    }
    return 0;
}

/* ---- NEXT-4: backward aggregation ----------------------------- */

/* GCN backward (the training workload of Eq. 1): the forward layer
 * is Y = M X with M[v,u] = sum over edges u->v of c_in(v) w_e c_out(u), so
 *   dX = M^T dY,  dX[u,f] = sum_{edges e: u -> v} c_in(v) w_e c_out(u) dY[v,f].
 * Written as the plain scatter over the forward CSR (no transposed CSR), fp64.
 * dX and A are [n_src x F] (all source rows). */
int oracle_gcn_backward(int64_t n_dst, int64_t n_src, const int64_t *rowptr,
                        const int32_t *colidx, const float *ew, const float *dY,
                        int64_t F, int64_t lddy, int norm, double *dX, double *A)
{
    if (norm < 0 || norm > 2 || F < 0 || lddy < F)
        return -1;
    int64_t nnz = rowptr[n_dst];
    int32_t *out_deg = (int32_t *)malloc(sizeof(int32_t) * (size_t)(n_src > 0 ? n_src : 1));
    if (!out_deg)
        return -1;
    oracle_out_degree(n_src, nnz, colidx, out_deg);
    for (int64_t i = 0; i < n_src * F; ++i) {
        dX[i] = 0.0;
        if (A)
            A[i] = 0.0;
    }
    for (int64_t v = 0; v < n_dst; ++v) {
        int64_t deg = rowptr[v + 1] - rowptr[v];
        double dclamp = (double)(deg > 1 ? deg : 1);
        double c_in = norm == ORACLE_NORM_RIGHT ? 1.0 / dclamp
                      : norm == ORACLE_NORM_BOTH ? 1.0 / sqrt(dclamp) : 1.0;
        for (int64_t e = rowptr[v]; e < rowptr[v + 1]; ++e) {
            int64_t u = colidx[e];
            double w = ew ? (double)ew[e] : 1.0;
            double c_out = 1.0;
            if (norm == ORACLE_NORM_BOTH) {
                int32_t od = out_deg[u];
                c_out = 1.0 / sqrt((double)(od > 1 ? od : 1));
            }
            double coef = c_in * w * c_out;
            for (int64_t f = 0; f < F; ++f) {
                double term = coef * (double)dY[v * lddy + f];
                dX[u * F + f] += term;
                if (A)
                    A[u * F + f] += fabs(term);
            }
        }
    }
    free(out_deg);
    return 0;
}

/* GIN backward: Y = (1+eps) X[v] + sum_e w_e X[u]  =>
 *   dX[u,f] = (1+eps) dY[u,f] + sum_{edges e: u -> v} w_e dY[v,f]
 * (square graph, n_dst = n_src). */
int oracle_gin_backward(int64_t n, const int64_t *rowptr, const int32_t *colidx,
                        const float *ew, const float *dY, int64_t F, int64_t lddy,
                        double eps, double *dX, double *A)
{
    if (F < 0 || lddy < F)
        return -1;
    for (int64_t u = 0; u < n; ++u)
        for (int64_t f = 0; f < F; ++f) {
            double t = (1.0 + eps) * (double)dY[u * lddy + f];
            dX[u * F + f] = t;
            if (A)
                A[u * F + f] = fabs(t);
        }
    for (int64_t v = 0; v < n; ++v)
        for (int64_t e = rowptr[v]; e < rowptr[v + 1]; ++e) {
            int64_t u = colidx[e];
            double w = ew ? (double)ew[e] : 1.0;
            for (int64_t f = 0; f < F; ++f) {
                double term = w * (double)dY[v * lddy + f];
                dX[u * F + f] += term;
                if (A)
                    A[u * F + f] += fabs(term);
            }
        }
    return 0;
}

/* GAT backward (single head; the training workload of the attention layer,
 * P:1001-1007, Velickovic [43]).  Forward, per destination v with in-edges e
 * (source u = colidx[e]):  t_e = el[u] + er[v],  s_e = LeakyReLU(t_e),
 * alpha_e = softmax over the in-edges of v of s_e,  Y[v] = sum_e alpha_e X[u].
 * Given dY, the chain rule written out step by step:
 *   g_e   = sum_f dY[v,f] X[u,f]                 (dL/dalpha_e)
 *   S_v   = sum_e alpha_e g_e
 *   ds_e  = alpha_e (g_e - S_v)                  (softmax Jacobian)
 *   dt_e  = ds_e * (t_e >= 0 ? 1 : slope)        (LeakyReLU, reading R6)
 *   dX[u,f] += alpha_e dY[v,f];  del[u] += dt_e;  der[v] += dt_e.
 * Bound terms (sum |terms|, for the parity criterion): G_e = sum_f |dY X|,
 * B_e = |slope_e| alpha_e (G_e + sum_e' alpha_e' G_e') for dt_e, and
 * |alpha_e dY[v,f]| for dX.  dX, AdX: [n_src x F]; del, Adel: [n_src];
 * der, Ader: [n_dst].  Two-pass softmax as in oracle_gat. */
int oracle_gat_backward(int64_t n_dst, int64_t n_src, const int64_t *rowptr,
                        const int32_t *colidx, const float *X, int64_t ldx,
                        const float *el, const float *er, double slope,
                        const float *dY, int64_t F, int64_t lddy,
                        double *dX, double *AdX, double *del, double *Adel,
                        double *der, double *Ader)
{
    if (F < 0 || ldx < F || lddy < F)
        return -1;
    for (int64_t i = 0; i < n_src * F; ++i) {
        dX[i] = 0.0;
        AdX[i] = 0.0;
    }
    for (int64_t u = 0; u < n_src; ++u) {
        del[u] = 0.0;
        Adel[u] = 0.0;
    }
    for (int64_t v = 0; v < n_dst; ++v) {
        int64_t e0 = rowptr[v], e1 = rowptr[v + 1];
        int64_t d = e1 - e0;
        der[v] = 0.0;
        Ader[v] = 0.0;
        if (d == 0)
            continue;
        double *alpha = (double *)malloc(sizeof(double) * (size_t)d);
        double *g = (double *)malloc(sizeof(double) * (size_t)d);
        double *G = (double *)malloc(sizeof(double) * (size_t)d);
        if (!alpha || !g || !G) {
            free(alpha); free(g); free(G);
            return -1;
        }
        double er_v = (double)er[v];
        /* forward softmax, two passes (as oracle_gat) */
        double m = -INFINITY;
        for (int64_t e = e0; e < e1; ++e) {
            double s = leaky_relu((double)el[colidx[e]] + er_v, slope);
            alpha[e - e0] = s;
            if (s > m)
                m = s;
        }
        double z = 0.0;
        for (int64_t k = 0; k < d; ++k)
            z += exp(alpha[k] - m);
        for (int64_t k = 0; k < d; ++k)
            alpha[k] = exp(alpha[k] - m) / z;
        /* g_e, S_v */
        double S = 0.0, SA = 0.0;
        for (int64_t e = e0; e < e1; ++e) {
            int64_t u = colidx[e];
            double gg = 0.0, GG = 0.0;
            for (int64_t f = 0; f < F; ++f) {
                double t = (double)dY[v * lddy + f] * (double)X[u * ldx + f];
                gg += t;
                GG += fabs(t);
            }
            g[e - e0] = gg;
            G[e - e0] = GG;
            S += alpha[e - e0] * gg;
            SA += alpha[e - e0] * GG;
        }
        for (int64_t e = e0; e < e1; ++e) {
            int64_t u = colidx[e];
            double a = alpha[e - e0];
            double t = (double)el[u] + er_v;
            double lr = t >= 0.0 ? 1.0 : slope;
            double dt = a * (g[e - e0] - S) * lr;
            double bt = fabs(lr) * a * (G[e - e0] + SA);
            der[v] += dt;
            Ader[v] += bt;
            del[u] += dt;
            Adel[u] += bt;
            for (int64_t f = 0; f < F; ++f) {
                double term = a * (double)dY[v * lddy + f];
                dX[u * F + f] += term;
                AdX[u * F + f] += fabs(term);
            }
        }
        free(alpha); free(g); free(G);
    }
    return 0;
}

/* NEXT-3: the next GAT layer's attention terms of a layer output (after the
 * epilogue), el[v] = sum_f Y[v,f] a[f]  (Velickovic [43]: a^T [W h_i || W h_j]
 * splits into a per-source and a per-destination dot product).
 * Y is fp32 [n_rows x ldy] (the previous stage's output, reading R22);
 * out, A: [n_rows] (A = sum |terms|). */
int oracle_project(int64_t n_rows, int64_t F, const float *Y, int64_t ldy,
                   const float *a, double *out, double *A)
{
    if (F < 0 || ldy < F)
        return -1;
    for (int64_t v = 0; v < n_rows; ++v) {
        double s = 0.0, b = 0.0;
        for (int64_t f = 0; f < F; ++f) {
            double t = (double)Y[v * ldy + f] * (double)a[f];
            s += t;
            b += fabs(t);
        }
        out[v] = s;
        if (A)
            A[v] = b;
    }
    return 0;
}

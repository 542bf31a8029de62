// panel.cuh -- fused column-wise panel factorization run by one CTA
// (irrGETF2, §IV-E: irrIAMAX -> irrSWAP -> irrSCAL -> irrGER fused in
// one kernel when the panel fits in shared memory).
//
// Two barriers per column: the rank-1 update of column c also produces the
// per-warp arg-max partials of column c+1 (and its diagonal value), so the
// next pivot is known right after the barrier without another pass.
#pragma once
#include "irr_internal.cuh"

namespace irr {

struct PanelScratch {
    unsigned long long key[32];
    int row[32];
    double val[32];
    double diag;
};

// P: column-major with leading dimension ldp (shared or global memory).
// Active rows [r0, rend); panel columns [c0, c0 + ib); the diagonal of panel
// column c is row r0 + c.  Row interchanges are applied across the columns
// [sw_lo, sw_hi) of P.  piv[c] receives the (P-relative) pivot row of column
// c0 + c.  Returns the 1-based local column of the first exact zero pivot, or 0
// (uniform over the CTA).  Must be called by all NT threads.
template <int NT>
__device__ int panel_getf2(double *P, int ldp, int r0, int rend, int c0, int ib, int sw_lo, int sw_hi, int *piv,
                           PanelScratch &sc) {
    constexpr int NW = NT / 32;
    const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
    int zero_at = 0;
    // ---- arg-max partials of the first panel column
    {
        unsigned long long bk = 0;
        int br = -1;
        double bv = 0.0;
        for (int r = r0 + tid; r < rend; r += NT) {
            double v = P[r + (size_t)c0 * ldp];
            unsigned long long k = dkey(fabs(v));
            if (br < 0 || k > bk) { bk = k; br = r; bv = v; }
            if (r == r0) sc.diag = v;
        }
        unsigned long long wk;
        int wr;
        warp_argmax(br >= 0, bk, br, wk, wr);
        unsigned wl = __ballot_sync(FULL, br >= 0 && br == wr);
        double wv = __shfl_sync(FULL, bv, wl ? __ffs(wl) - 1 : 0);
        if (lane == 0) { sc.key[warp] = wk; sc.row[warp] = wr; sc.val[warp] = wv; }
    }
    __syncthreads();
    for (int c = 0; c < ib; ++c) {
        const int col = c0 + c, dr = r0 + c;
        // ---- final arg-max over the warp partials (every thread, redundantly)
        unsigned long long bk = 0;
        int p = -1;
        double pv = 0.0;
#pragma unroll
        for (int w = 0; w < NW; ++w) {
            int rr = sc.row[w];
            if (rr < 0) continue;
            unsigned long long kk = sc.key[w];
            if (p < 0 || kk > bk || (kk == bk && rr < p)) { bk = kk; p = rr; pv = sc.val[w]; }
        }
        const double dold = sc.diag;
        if (tid == 0) piv[c] = p;
        // ---- interchange rows dr <-> p across [sw_lo, sw_hi), scale column col
        if (pv != 0.0) {
            if (p != dr) {
                for (int cc = sw_lo + tid; cc < sw_hi; cc += NT) {
                    if (cc == col) continue;
                    double t = P[dr + (size_t)cc * ldp];
                    P[dr + (size_t)cc * ldp] = P[p + (size_t)cc * ldp];
                    P[p + (size_t)cc * ldp] = t;
                }
            }
            PivotScale s(pv);
            for (int r = dr + 1 + tid; r < rend; r += NT) {
                double v = (r == p) ? dold : P[r + (size_t)col * ldp];
                P[r + (size_t)col * ldp] = s(v);
            }
            if (tid == 0) P[dr + (size_t)col * ldp] = pv;
        } else if (zero_at == 0) {
            zero_at = c + 1;  // all candidates are exactly 0: p == dr, no swap, no scaling
        }
        __syncthreads();
        // ---- rank-1 update of the panel columns right of col; arg-max of col+1
        const int cend = c0 + ib;
        const bool more = c + 1 < ib;
        unsigned long long nk = 0;
        int nr = -1;
        double nv = 0.0;
        for (int r = dr + 1 + tid; r < rend; r += NT) {
            const double l = P[r + (size_t)col * ldp];
            for (int cc = col + 1; cc < cend; ++cc)
                P[r + (size_t)cc * ldp] = fma(-l, P[dr + (size_t)cc * ldp], P[r + (size_t)cc * ldp]);
            if (more) {
                double v = P[r + (size_t)(col + 1) * ldp];
                unsigned long long k = dkey(fabs(v));
                if (nr < 0 || k > nk) { nk = k; nr = r; nv = v; }
                if (r == dr + 1) sc.diag = v;
            }
        }
        if (more) {
            unsigned long long wk;
            int wr;
            warp_argmax(nr >= 0, nk, nr, wk, wr);
            unsigned wl = __ballot_sync(FULL, nr >= 0 && nr == wr);
            double wv = __shfl_sync(FULL, nv, wl ? __ffs(wl) - 1 : 0);
            if (lane == 0) { sc.key[warp] = wk; sc.row[warp] = wr; sc.val[warp] = wv; }
        }
        __syncthreads();
    }
    return zero_at;
}

}  // namespace irr

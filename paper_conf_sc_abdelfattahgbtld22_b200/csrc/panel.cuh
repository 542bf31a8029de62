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

// Composition of the ib interchanges of one panel (rows j .. j+ib-1) on an
// index list: position j+t receives row top_src[t]; position bot_pos[b] (below
// the panel block) receives row bot_src[b].
struct SwapPlan {
    int top_src[64];
    int piv[64];
    int bot_pos[64], bot_src[64];
    int nbot;
};

struct PanelScratch {
    unsigned long long key[32];
    int row[32];
    double val[32];
    double diag;
};

// ---------------------------------------------------------------------------
// Register-resident panel, ONE barrier per column (panel_regs).
//
// Thread t owns panel rows t, t+NT, ... (RPT of them), each held in registers
// in shift-register form: a[q][0] is always the current column, and the
// rank-1 update is fused with the shift, a[q][k] <- a[q][k+1] - l u[k+1]
// (as in tier S).  Rows never move: an interchange relabels positions.  Per
// column, every warp publishes its arg-max partial TOGETHER with the values
// of its candidate row (double-buffered slots), so after the single barrier
// every thread knows the pivot and already has the pivot row.  The factored
// panel is assembled in shared memory in LAPACK order as values become final:
// U row c at step c, each L value at its row's current position, and the
// already-final L columns of positions c and pmin are exchanged (one thread
// per column) -- the "rehearsal" of P:L192 applied on the fly.
#ifdef IRR_PANEL_TIMING  // tools/panel_bench.cu only
__device__ unsigned long long g_ptime[8];
__shared__ unsigned long long s_ptime[8];
#define PT(k)                                                                                  \
    if (threadIdx.x == 0) {                                                                    \
        long long t_ = clock64();                                                              \
        s_ptime[k] += (unsigned long long)(t_ - pt0_);                                         \
        pt0_ = t_;                                                                             \
    }
#define PT0 long long pt0_ = clock64();
#else
#define PT(k)
#define PT0
#endif

template <int NW, int NBP>
struct PanelRegScratch {
    double row[2][NW][NBP];  // first: 16-byte aligned for the pair stores; row[.][w][0] = signed candidate
    unsigned long long key[2][NW];
    double rcp[2][NW];
    int pos[2][NW];
};

// One column step of panel_regs on the W active (shifted) columns.
template <int NT, int RPT, int NBP, int W>
__device__ __forceinline__ void preg_step(double (&a)[RPT][NBP], int (&pos)[RPT], int c, double *P, int ldp, int rows,
                                          int ib, int *piv, PanelRegScratch<NT / 32, NBP> &sc, int &zero_at) {
    constexpr int NW = NT / 32;
    const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
    const int par = c & 1;
    PT0
    // ---- thread / warp candidates of column c (positions >= c)
    unsigned long long bk = 0;
    int bp = 0x7fffffff, bq = -1;
#pragma unroll
    for (int q = 0; q < RPT; ++q) {
        const int r = tid + NT * q;
        if (r < rows && pos[q] >= c) {
            const unsigned long long k = dkey(fabs(a[q][0]));
            if (bq < 0 || k > bk || (k == bk && pos[q] < bp)) { bk = k; bp = pos[q]; bq = q; }
        }
    }
    // speculative reciprocal of this thread's candidate (published by the winner)
    double cv = a[0][0];
#pragma unroll
    for (int q = 1; q < RPT; ++q)
        if (bq == q) cv = a[q][0];
    const double myr = fast_rcp(cv);
    const int wl = warp_argmax_lane(bq >= 0, bk, bp);
    const unsigned long long wk = bk;  // the winner's own key / position
    const int wp = bp;
    const unsigned wm = wl < 0 ? 0u : (1u << wl);
    PT(0)
    if (wm == 0) {
        if (lane == 0) sc.pos[par][warp] = -1;
    } else if (lane == __ffs(wm) - 1) {
        // publish the candidate row with the partial (no selects: one branch per row slot)
        sc.key[par][warp] = wk;
        sc.pos[par][warp] = wp;
        sc.rcp[par][warp] = myr;
        double *dst = sc.row[par][warp];
#pragma unroll
        for (int q = 0; q < RPT; ++q) {
            if (bq == q) {
#pragma unroll
                for (int k = 0; k < W; k += 2)
                    *reinterpret_cast<double2 *>(dst + k) = make_double2(a[q][k], a[q][k + 1]);
            }
        }
    }
    PT(1)
    __syncthreads();
    PT(2)
    // ---- the pivot: every thread reduces the NW partials (all loads first)
    int pp[NW];
    unsigned long long kk[NW];
#pragma unroll
    for (int w = 0; w < NW; ++w) { pp[w] = sc.pos[par][w]; kk[w] = sc.key[par][w]; }
    int wbest = -1, pmin = 0x7fffffff;
    unsigned long long kb = 0;
#pragma unroll
    for (int w = 0; w < NW; ++w) {
        const int p = pp[w];
        if (p < 0) continue;
        if (wbest < 0 || kk[w] > kb || (kk[w] == kb && p < pmin)) { kb = kk[w]; pmin = p; wbest = w; }
    }
    const double *u = sc.row[par][wbest];
    const double pv = u[0];
    if (tid == 0) piv[c] = pmin;
    PT(3)
    // ---- final pieces of the result: swap the L columns < c of positions c
    //      and pmin, write U row c
    if (pmin != c && tid < c) {
        const double x = P[c + tid * ldp], y = P[pmin + tid * ldp];
        P[c + tid * ldp] = y;
        P[pmin + tid * ldp] = x;
    }
    if (tid < ib - c) P[c + (c + tid) * ldp] = u[tid];
#pragma unroll
    for (int q = 0; q < RPT; ++q) {
        if (pos[q] == c) pos[q] = pmin;
        else if (pos[q] == pmin) pos[q] = c;
    }
    if (pv == 0.0 && zero_at == 0) zero_at = c + 1;  // no interchange (pmin == c), no scaling
    const double rcp = sc.rcp[par][wbest];  // 0: divide (|pv| < sfmin or 1/pv subnormal)
    PT(4)
    // ---- scale + rank-1 update + shift of my rows below position c
    double lq[RPT];
    bool act[RPT];
#pragma unroll
    for (int q = 0; q < RPT; ++q) {
        act[q] = (tid + NT * q < rows) && pos[q] > c;
        double l = a[q][0];
        if (pv != 0.0) l = (rcp != 0.0) ? l * rcp : l / pv;
        lq[q] = l;
    }
    // a[e-1] <- a[e] - l u[e], e ascending; u streamed in 16-byte loads,
    // eight values live at a time (register budget of the L1 kernel)
    constexpr int CH = W < 8 ? W : 8;
#pragma unroll
    for (int e0 = 0; e0 < W; e0 += CH) {
        double uu[CH];
#pragma unroll
        for (int k = 0; k < CH; k += 2) {
            const double2 t = *reinterpret_cast<const double2 *>(u + e0 + k);
            uu[k] = t.x;
            uu[k + 1] = t.y;
        }
#pragma unroll
        for (int q = 0; q < RPT; ++q) {
            if (act[q]) {
#pragma unroll
                for (int k = 0; k < CH; ++k)
                    if (e0 + k >= 1) a[q][e0 + k - 1] = fma(-lq[q], uu[k], a[q][e0 + k]);
            }
        }
    }
#pragma unroll
    for (int q = 0; q < RPT; ++q) {
        if (act[q]) {
            a[q][W - 1] = 0.0;
            P[pos[q] + c * ldp] = lq[q];
        }
    }
    PT(5)
}

// P: shared-memory panel, rows x ib, column-major (ldp); rows <= NT * RPT,
// ib <= NBP.  On return P holds L\U of the panel in LAPACK row order and
// piv[c] the 0-based pivot position of column c.  Returns the 1-based column of
// the first exact zero pivot, or 0.  All NT threads must call it.  The active
// width W shrinks NBP -> NBP/2 -> ... -> 4 with the remaining columns.
template <int NT, int RPT, int NBP>
__device__ int panel_regs(double *P, int ldp, int rows, int ib, int *piv, PanelRegScratch<NT / 32, NBP> &sc,
                          SwapPlan *plan = nullptr, int row0 = 0) {
    const int tid = threadIdx.x;
    if (plan && tid == 0) plan->nbot = 0;
    double a[RPT][NBP];
    int pos[RPT];
#pragma unroll
    for (int q = 0; q < RPT; ++q) {
        const int r = tid + NT * q;
        pos[q] = r;
#pragma unroll
        for (int k = 0; k < NBP; ++k) a[q][k] = (r < rows && k < ib) ? P[r + k * ldp] : 0.0;
    }
    __syncthreads();  // P is overwritten with the result from here on
    int zero_at = 0, c = 0;
    if (NBP >= 64)
        for (; c < ib && ib - c > 32; ++c) preg_step<NT, RPT, NBP, (NBP >= 64 ? 64 : NBP)>(a, pos, c, P, ldp, rows, ib, piv, sc, zero_at);
    if (NBP >= 32)
        for (; c < ib && ib - c > 16; ++c) preg_step<NT, RPT, NBP, (NBP >= 32 ? 32 : NBP)>(a, pos, c, P, ldp, rows, ib, piv, sc, zero_at);
    if (NBP >= 16)
        for (; c < ib && ib - c > 8; ++c) preg_step<NT, RPT, NBP, (NBP >= 16 ? 16 : NBP)>(a, pos, c, P, ldp, rows, ib, piv, sc, zero_at);
    for (; c < ib && ib - c > 4; ++c) preg_step<NT, RPT, NBP, 8>(a, pos, c, P, ldp, rows, ib, piv, sc, zero_at);
    for (; c < ib; ++c) preg_step<NT, RPT, NBP, 4>(a, pos, c, P, ldp, rows, ib, piv, sc, zero_at);
    if (plan) {
        // the interchange plan straight from the final positions (parallel;
        // replaces composing the ib interchanges serially): a row ending in
        // the top block names its source; a row pushed below it came from the
        // top block and becomes a (pos, src) pair.  Absolute rows = row0 + .
#pragma unroll
        for (int q = 0; q < RPT; ++q) {
            const int r = tid + NT * q;
            if (r < rows) {
                const int p = pos[q];
                if (p < ib) {
                    plan->top_src[p] = row0 + r;
                } else if (p != r) {
                    const int b = atomicAdd(&plan->nbot, 1);
                    plan->bot_pos[b] = row0 + p;
                    plan->bot_src[b] = row0 + r;
                }
            }
        }
    }
    __syncthreads();
    return zero_at;
}

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
            // batches of 8 columns: all loads issued before the dependent
            // stores (the element-wise form serialised on possible aliasing)
            for (int q0 = col + 1; q0 < cend; q0 += 8) {
                double u[8], v[8];
#pragma unroll
                for (int q = 0; q < 8; ++q) {
                    const bool ok = q0 + q < cend;
                    u[q] = ok ? P[dr + (size_t)(q0 + q) * ldp] : 0.0;
                    v[q] = ok ? P[r + (size_t)(q0 + q) * ldp] : 0.0;
                }
#pragma unroll
                for (int q = 0; q < 8; ++q)
                    if (q0 + q < cend) P[r + (size_t)(q0 + q) * ldp] = fma(-l, u[q], v[q]);
            }
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

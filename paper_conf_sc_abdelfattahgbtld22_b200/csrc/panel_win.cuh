// panel_win.cuh -- register-resident panel for TALL panels (rows up to
// NT * RPT, panel width ib <= 64) working directly on the matrix in global
// memory: irrGETF2 (§IV-E) for the grid-wide tier, where a 1024 x 32
// panel would need the whole register file (or 256 KB of shared memory).
//
// Column-blocked ("windowed"): each thread holds only a WB-wide window of its
// RPT rows in registers (shift form, as panel_regs: a[q][0] is the current
// column, one CTA barrier per column).  The window advances left-looking: the
// next WB columns are read fresh from HBM and brought up to date with the L
// and U computed so far -- a unit-lower triangular solve for the pivot rows and
// a rank-b0 update for the others.  Rows never move while the panel runs:
//   * every L value is written at its row's ORIGINAL index (no interchange of
//     finished L columns, no read-modify-write of global memory on the chain);
//   * U rows are assembled in shared memory (Us);
//   * one permutation at the end writes L\U in LAPACK row order, touching only
//     the <= 2 ib rows that moved, and emits the interchange plan.
#pragma once
#include "panel.cuh"

namespace irr {

constexpr int PW_WBMAX = 16;

template <int NW, int NBX = 64>  // NBX: largest panel width (<= 64)
struct PanelWinSmem {
    double Us[NBX * (NBX + 1)];  // U rows: Us[p][k], k >= p
    double Lb[NBX * (NBX + 1)];  // L of the pivot rows: Lb[p][s], s < p
    double Ds[NBX * (NBX + 1)];  // L of the rows pushed below the panel block (end)
    double row[2][NW][PW_WBMAX];  // published candidate rows (double-buffered)
    unsigned long long key[2][NW];
    double rcp[2][NW];
    int pos[2][NW], orig[2][NW];
    int srcpos[NBX];  // original row now at pivot position p
    SwapPlan plan;
};

// One column step on the W active (shifted) columns of the window ending at
// column bend.  Same protocol as preg_step; differs in where results go.
template <int NT, int RPT, int WB, int W, int NBX>
__device__ __forceinline__ void pwin_step(double (&a)[RPT][WB], int (&pos)[RPT], int c, int bend, double *gP,
                                          long ld, int rows, int *piv, PanelWinSmem<NT / 32, NBX> &sm, int &zero_at) {
    constexpr int NW = NT / 32;
    const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
    const int par = c & 1;
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
    if (wm == 0) {
        if (lane == 0) sm.pos[par][warp] = -1;
    } else if (lane == __ffs(wm) - 1) {
        sm.key[par][warp] = wk;
        sm.pos[par][warp] = wp;
        sm.rcp[par][warp] = myr;
        sm.orig[par][warp] = tid + NT * bq;
        double *dst = sm.row[par][warp];
#pragma unroll
        for (int q = 0; q < RPT; ++q) {
            if (bq == q) {
#pragma unroll
                for (int k = 0; k < W; k += 2)
                    *reinterpret_cast<double2 *>(dst + k) = make_double2(a[q][k], a[q][k + 1]);
            }
        }
    }
    __syncthreads();
    int pp[NW];
    unsigned long long kk[NW];
#pragma unroll
    for (int w = 0; w < NW; ++w) { pp[w] = sm.pos[par][w]; kk[w] = sm.key[par][w]; }
    int wbest = -1, pmin = 0x7fffffff;
    unsigned long long kb = 0;
#pragma unroll
    for (int w = 0; w < NW; ++w) {
        const int p = pp[w];
        if (p < 0) continue;
        if (wbest < 0 || kk[w] > kb || (kk[w] == kb && p < pmin)) { kb = kk[w]; pmin = p; wbest = w; }
    }
    const double *u = sm.row[par][wbest];
    const double pv = u[0];
    if (tid == 0) {
        piv[c] = pmin;
        sm.srcpos[c] = sm.orig[par][wbest];
    }
    if (tid < bend - c) sm.Us[c * (NBX + 1) + c + tid] = u[tid];  // U row c inside the window
#pragma unroll
    for (int q = 0; q < RPT; ++q) {
        if (pos[q] == c) pos[q] = pmin;
        else if (pos[q] == pmin) pos[q] = c;
    }
    if (pv == 0.0 && zero_at == 0) zero_at = c + 1;  // no interchange (pmin == c), no scaling
    const double rcp = sm.rcp[par][wbest];  // 0: divide (|pv| < sfmin or 1/pv subnormal)
    double lq[RPT];
    bool act[RPT];
#pragma unroll
    for (int q = 0; q < RPT; ++q) {
        act[q] = (tid + NT * q < rows) && pos[q] > c;
        double l = a[q][0];
        if (pv != 0.0) l = (rcp != 0.0) ? l * rcp : l / pv;
        lq[q] = l;
    }
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
            gP[tid + NT * q + (size_t)c * ld] = lq[q];  // L at the ORIGINAL row index
        }
    }
}

// gP: the panel's top-left element (global), rows x ib, column-major (ld);
// rows <= NT * RPT, ib <= 64, WB <= PW_WBMAX.  On return gP holds L\U of the
// panel in LAPACK row order, piv[c] the 0-based pivot position of column c,
// and sm.plan the interchange plan (relative rows).  Returns the 1-based column
// of the first exact zero pivot, or 0.  All NT threads must call it.
template <int NT, int RPT, int WB, int NBX = 64>
__device__ int panel_win(double *gP, long ld, int rows, int ib, int *piv, PanelWinSmem<NT / 32, NBX> &sm) {
    constexpr int NW = NT / 32;
    const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
    double a[RPT][WB];
    int pos[RPT];
#pragma unroll
    for (int q = 0; q < RPT; ++q) pos[q] = tid + NT * q;
    if (tid == 0) sm.plan.nbot = 0;
    int zero_at = 0;
    int b0 = 0;
    for (; b0 < ib; b0 += WB) {
        const int bend = imin(ib, b0 + WB);
        const int bw = bend - b0;
        // ---- the window's original values (coalesced: lanes over rows)
#pragma unroll
        for (int q = 0; q < RPT; ++q) {
            const int r = tid + NT * q;
#pragma unroll
            for (int k = 0; k < WB; ++k) a[q][k] = (r < rows && k < bw) ? gP[r + (size_t)(b0 + k) * ld] : 0.0;
        }
        if (b0 > 0) {
            // (i) L of the previous window's pivot rows -> Lb; (ii) their window
            // values -> Us (to be solved).  Warps over columns, lanes over rows.
            const int p0 = b0 - WB;
            for (int s = warp; s < b0; s += NW)
                for (int p = imax(p0, s + 1) + lane; p < b0; p += 32)
                    sm.Lb[p * (NBX + 1) + s] = gP[sm.srcpos[p] + (size_t)s * ld];
            for (int k = warp; k < bw; k += NW)
                for (int p = lane; p < b0; p += 32) sm.Us[p * (NBX + 1) + b0 + k] = gP[sm.srcpos[p] + (size_t)(b0 + k) * ld];
            __syncthreads();
            // (iii) U[0:b0, window] = L11^{-1} U[0:b0, window]: warp per column,
            // the column in registers (2 rows per lane), x_s by shuffle
            for (int k = warp; k < bw; k += NW) {
                double x0 = lane < b0 ? sm.Us[lane * (NBX + 1) + b0 + k] : 0.0;
                double x1 = lane + 32 < b0 ? sm.Us[(lane + 32) * (NBX + 1) + b0 + k] : 0.0;
                for (int s = 0; s < b0 - 1; ++s) {
                    const double xs = __shfl_sync(FULL, s < 32 ? x0 : x1, s & 31);
                    if (lane > s && lane < b0) x0 = fma(-sm.Lb[lane * (NBX + 1) + s], xs, x0);
                    if (lane + 32 > s && lane + 32 < b0) x1 = fma(-sm.Lb[(lane + 32) * (NBX + 1) + s], xs, x1);
                }
                if (lane < b0) sm.Us[lane * (NBX + 1) + b0 + k] = x0;
                if (lane + 32 < b0) sm.Us[(lane + 32) * (NBX + 1) + b0 + k] = x1;
            }
            __syncthreads();
            // (iv) rows still below the pivots: a -= L(r, 0:b0) U(0:b0, window)
            bool live[RPT];
#pragma unroll
            for (int q = 0; q < RPT; ++q) live[q] = (tid + NT * q < rows) && pos[q] >= b0;
            for (int s = 0; s < b0; ++s) {
                double l[RPT];
#pragma unroll
                for (int q = 0; q < RPT; ++q) l[q] = live[q] ? gP[tid + NT * q + (size_t)s * ld] : 0.0;
                const double *us = sm.Us + s * (NBX + 1) + b0;
#pragma unroll
                for (int k = 0; k < WB; ++k) {
                    const double uk = us[k];
#pragma unroll
                    for (int q = 0; q < RPT; ++q) a[q][k] = fma(-l[q], uk, a[q][k]);
                }
            }
        }
        // ---- column steps; the active width halves with the window's remaining columns
        int c = b0;
        if (WB >= 16)
            for (; c < bend && bend - c > 8; ++c)
                pwin_step<NT, RPT, WB, (WB >= 16 ? 16 : WB), NBX>(a, pos, c, bend, gP, ld, rows, piv, sm, zero_at);
        if (WB >= 8)
            for (; c < bend && bend - c > 4; ++c)
                pwin_step<NT, RPT, WB, (WB >= 8 ? 8 : WB), NBX>(a, pos, c, bend, gP, ld, rows, piv, sm, zero_at);
        for (; c < bend; ++c) pwin_step<NT, RPT, WB, (WB >= 4 ? 4 : WB), NBX>(a, pos, c, bend, gP, ld, rows, piv, sm, zero_at);
        __syncthreads();
    }
    // ---- the permutation: L of the last window's pivots, and of the rows
    //      pushed below the block (owner threads), plus the plan
    {
        const int p0 = ((ib - 1) / WB) * WB;
        for (int s = warp; s < ib; s += NW)
            for (int p = imax(p0, s + 1) + lane; p < ib; p += 32)
                sm.Lb[p * (NBX + 1) + s] = gP[sm.srcpos[p] + (size_t)s * ld];
    }
#pragma unroll
    for (int q = 0; q < RPT; ++q) {
        const int r = tid + NT * q;
        if (r < rows) {
            const int p = pos[q];
            if (p < ib) {
                sm.plan.top_src[p] = r;
            } else if (p != r) {
                const int b = atomicAdd(&sm.plan.nbot, 1);
                sm.plan.bot_pos[b] = p;
                sm.plan.bot_src[b] = r;
                for (int s = 0; s < ib; ++s) sm.Ds[b * (NBX + 1) + s] = gP[r + (size_t)s * ld];
            }
        }
    }
    __syncthreads();
    const int nbot = sm.plan.nbot;
    for (int s = warp; s < ib; s += NW) {
        for (int p = lane; p < ib; p += 32)
            gP[p + (size_t)s * ld] = s < p ? sm.Lb[p * (NBX + 1) + s] : sm.Us[p * (NBX + 1) + s];
        for (int b = lane; b < nbot; b += 32) gP[sm.plan.bot_pos[b] + (size_t)s * ld] = sm.Ds[b * (NBX + 1) + s];
    }
    __syncthreads();
    return zero_at;
}

}  // namespace irr

// lu_large.cu -- tier L: blocked right-looking LU with partial pivoting on
// the matrices too large for one shared-memory tile.
//
// The algorithm is the paper's (Fig. 1): per panel of nb columns,
//   a4.1 panel       fused irrGETF2 on the (m_i - j) x ib panel, staged in
//                    shared memory, interchanges inside the panel
//   a4.2+a4.3 swap   the panel's row interchanges "rehearsed" on an index list
//                     and applied once per moved row to the left and
//                    right column blocks; the right block is solved in the
//                    same pass: U12 <- L11^-1 P A12 (irrLASWP + irrTRSM fused)
//   a4.4 gemm        A22 -= L21 U12 with the pipelined FP64 GEMM core
// in two execution shapes:
//   L1  (m <= 256 rows): ONE CTA per matrix runs every iteration of every step
//       back to back (persistent CTAs, dynamic matrix queue); the matrix stays
//       L2-resident between iterations, so HBM sees it about once, and there
//       is no inter-kernel synchronisation at all.  Three CTAs per SM overlap
//       one matrix's latency-bound panel with other matrices' GEMMs.
//   L2  (taller): the host loops over panel ITERATIONS of the largest matrix
//       (DCWI: each kernel infers full / partial / no work per
//       matrix) with grid-wide kernels per step, so a few huge fronts use the
//       whole GPU.
#include "gemm_big.cuh"
#include "panel.cuh"
#include "panel_win.cuh"
#include "sched.cuh"

namespace irr {

constexpr int P_NT = 512;
constexpr int NBMAX = 64;     // largest supported panel width
constexpr int SW_COLS = 128;  // columns per swap/TRSM chunk (one thread per column)
constexpr int SW_NT = 128;
constexpr int L1_NT = 128;    // threads of the CTA-per-matrix kernel (== G_NT == SW_NT)
static_assert(L1_NT == G_NT && L1_NT == SW_NT, "L1 composes the GEMM and swap pieces at one CTA size");

// ------------------------------------------------------------------ swap plan
// (SwapPlan is defined in panel.cuh: panel_regs can emit it directly.)

// The plan of one outer block of the two-level grid tier (up to
// NB_OUTER_MAX interchanges; same fields as SwapPlan).
struct OuterPlan {
    int top_src[NB_OUTER_MAX];
    int piv[NB_OUTER_MAX];
    int bot_pos[NB_OUTER_MAX], bot_src[NB_OUTER_MAX];
    int nbot;
};
static_assert(sizeof(OuterPlan) <= OUTER_PLAN_BYTES, "outer plan slot");

// One warp composes the interchanges held in sp.piv[0..ib) (0-based absolute
// rows).  Caller synchronises afterwards.
template <class Plan>
__device__ __forceinline__ void plan_swaps_core(int j, int ib, Plan &sp) {
    const int lane = threadIdx.x & 31;
    const int c1 = j + ib;
    for (int t = lane; t < ib; t += 32) sp.top_src[t] = j + t;
    int nbot = 0;
    __syncwarp();
    for (int t = 0; t < ib; ++t) {
        const int p = sp.piv[t];
        if (p == j + t) continue;
        if (p < c1) {
            if (lane == 0) {
                int x = sp.top_src[t];
                sp.top_src[t] = sp.top_src[p - j];
                sp.top_src[p - j] = x;
            }
        } else {
            int found = -1;
            for (int b0 = 0; b0 < nbot; b0 += 32) {
                int b = b0 + lane;
                unsigned mk = __ballot_sync(FULL, b < nbot && sp.bot_pos[b] == p);
                if (mk) { found = b0 + __ffs(mk) - 1; break; }
            }
            if (found < 0) {
                found = nbot++;
                if (lane == 0) { sp.bot_pos[found] = p; sp.bot_src[found] = p; }
            }
            if (lane == 0) {
                int x = sp.top_src[t];
                sp.top_src[t] = sp.bot_src[found];
                sp.bot_src[found] = x;
            }
        }
        __syncwarp();
    }
    if (lane == 0) sp.nbot = nbot;
}

// plan from ipiv[j .. j+ib) in global memory (1-based): one coalesced load
__device__ __forceinline__ void plan_swaps(const int *__restrict__ ip, int j, int ib, SwapPlan &sp) {
    if ((threadIdx.x >> 5) != 0) return;
    for (int t = threadIdx.x & 31; t < ib; t += 32) sp.piv[t] = ip[j + t] - 1;
    __syncwarp();
    plan_swaps_core(j, ib, sp);
}

// plan from pivots already in shared memory (0-based absolute rows)
__device__ __forceinline__ void plan_swaps_from(const int *piv_abs, int j, int ib, SwapPlan &sp) {
    if ((threadIdx.x >> 5) != 0) return;
    for (int t = threadIdx.x & 31; t < ib; t += 32) sp.piv[t] = piv_abs[t];
    __syncwarp();
    plan_swaps_core(j, ib, sp);
}

// x <- L11^-1 x for one column x (stride ldx in shared memory), unit lower L11
// column-major with leading dimension ldl, or, when ldl == 0, its strict lower
// triangle packed by columns (column s = rows s+1..ib-1 at s(2ib-s-1)/2).
// Shift-register form (as in tier S): v[0] is always the next solution
// entry, so the loop body is the same for every step (O(W) code, no local
// memory) and each step is W-1 independent FMAs, W shrinking 32 -> 4.
// trsm_col_step: one substitution step on the W leading registers (the
// remaining rows of the column fit in W: ib - s <= W).
template <int NBX, int W>
__device__ __forceinline__ void trsm_col_step(double (&v)[NBX], double *x, int ldx, int ib, int s,
                                              const double *L11, int ldl) {
    const double xs = v[0];
    x[s * ldx] = xs;
    // column s of L11 below the diagonal is contiguous in both layouts
    const double *Ls = L11 + (ldl ? s + 1 + s * ldl : (s * (2 * ib - s - 1)) / 2);
    const int cnt = ib - s - 1;
#pragma unroll
    for (int q = 0; q + 1 < W; ++q) {
        const double l = (q < cnt) ? Ls[q] : 0.0;
        v[q] = fma(-l, xs, v[q + 1]);
    }
    v[W - 1] = 0.0;
}

template <int NBX>
__device__ __forceinline__ void trsm_col_regs(double *x, int ldx, int ib, const double *L11, int ldl) {
    double v[NBX];
#pragma unroll
    for (int r = 0; r < NBX; ++r) v[r] = (r < ib) ? x[r * ldx] : 0.0;
    // the active width shrinks with the remaining rows (as in the panel):
    // about half the FMAs and L loads of a fixed-width sweep
    int s = 0;
    if (NBX >= 32)
        for (; ib - s > 16; ++s) trsm_col_step<NBX, (NBX >= 32 ? 32 : NBX)>(v, x, ldx, ib, s, L11, ldl);
    if (NBX >= 16)
        for (; ib - s > 8; ++s) trsm_col_step<NBX, (NBX >= 16 ? 16 : NBX)>(v, x, ldx, ib, s, L11, ldl);
    for (; ib - s > 4; ++s) trsm_col_step<NBX, (NBX >= 8 ? 8 : NBX)>(v, x, ldx, ib, s, L11, ldl);
    for (; s < ib; ++s) trsm_col_step<NBX, 4>(v, x, ldx, ib, s, L11, ldl);
}

// Apply the plan to W columns of one matrix given as a VIRTUAL range
// [vbeg, vbeg+W): virtual column v is real column v (v < jsplit) or v + shift
// (v >= jsplit), so one chunk can span the left block [0, j) and the right
// block [j+ib, n) (fewer gather/solve/scatter rounds).  Real columns >=
// solve_from also get U12 <- L11^-1 (rows j..j+ib-1), L11 in shared memory in
// the layouts of trsm_col_regs.  top / bot: shared buffers of nb x
// (SW_COLS+1).  SW_NT threads.
template <int COLS = SW_COLS, int LT = COLS + 1>
__device__ __forceinline__ void swap_chunk(double *__restrict__ gA, long ld, int j, int ib, int vbeg, int W,
                                           int jsplit, int shift, int solve_from, const SwapPlan &sp,
                                           const double *L11, int ldl, double *top, double *bot,
                                           unsigned long long *ph = nullptr) {
    const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
    long long tq = (ph && tid == 0) ? clock64() : 0;
#define SWAP_PHASE(k)                                                         \
    if (ph && tid == 0) {                                                     \
        long long t1 = clock64();                                             \
        atomicAdd(ph + (k), (unsigned long long)(t1 - tq));                   \
        tq = t1;                                                              \
    }
    constexpr int NWS = SW_NT / 32;
    const int nbot = sp.nbot;
    // warps over columns, lanes over the (<= 64) moved rows: no integer division
    for (int c = warp; c < W; c += NWS) {
        const int v = vbeg + c, col = v < jsplit ? v : v + shift;
        const double *gc = gA + (size_t)col * ld;
        for (int t = lane; t < ib; t += 32) cp_async8(&top[t * LT + c], gc + sp.top_src[t]);
        for (int b = lane; b < nbot; b += 32) cp_async8(&bot[b * LT + c], gc + sp.bot_src[b]);
    }
    cp_async_commit();
    cp_async_wait<0>();
    __syncthreads();
    SWAP_PHASE(5)
    if (tid < W) {
        const int v = vbeg + tid, col = v < jsplit ? v : v + shift;
        if (col >= solve_from) {
            // one thread per column, the column in registers (the smem
            // read-modify-write form was a serial LDS->DFMA->STS chain)
            if (ib <= 32) {
                trsm_col_regs<32>(top + tid, LT, ib, L11, ldl);
            } else {  // nb > 32 (tuning only): plain shared-memory substitution
                for (int s = 0; s < ib; ++s) {
                    const double x = top[s * LT + tid];
                    const double *Ls = L11 + (ldl ? s + 1 + s * ldl : (s * (2 * ib - s - 1)) / 2);
                    for (int r = s + 1; r < ib; ++r) top[r * LT + tid] = fma(-Ls[r - s - 1], x, top[r * LT + tid]);
                }
            }
        }
    }
    __syncthreads();
    SWAP_PHASE(6)
    for (int c = warp; c < W; c += NWS) {
        const int v = vbeg + c, col = v < jsplit ? v : v + shift;
        double *gc = gA + (size_t)col * ld;
        for (int t = lane; t < ib; t += 32) gc[j + t] = top[t * LT + c];
        for (int b = lane; b < nbot; b += 32) gc[sp.bot_pos[b]] = bot[b * LT + c];
    }
    __syncthreads();
    SWAP_PHASE(7)
#undef SWAP_PHASE
}

// L11 (ib x ib diagonal block at (j, j)) -> shared memory, column-major (ldl)
__device__ __forceinline__ void load_L11_async(double *L11, int ldl, const double *gA, long ld, int j, int ib) {
    const int lane = threadIdx.x & 31, nw = blockDim.x >> 5;
    for (int c = threadIdx.x >> 5; c < ib; c += nw)
        for (int r = lane; r < ib; r += 32) cp_async8(&L11[r + c * ldl], gA + j + r + (size_t)(j + c) * ld);
}

// trailing-update descriptor of one matrix at iteration j (false: no GEMM work)
__device__ __forceinline__ bool trailing_desc(double *A, long ld, int mi, int ni, int j, int nb, GemmDesc &d) {
    const int K = mi < ni ? mi : ni;
    d.m = 0; d.n = 0; d.k = 0;
    if (j >= K) return false;
    const int ib = K - j < nb ? K - j : nb;
    const int c1 = j + ib;
    if (c1 >= mi || c1 >= ni) return false;
    d.A = A + c1 + (size_t)j * ld; d.lda = ld; d.ta = 0;
    d.B = A + j + (size_t)c1 * ld; d.ldb = ld; d.tb = 0;
    d.C = A + c1 + (size_t)c1 * ld; d.ldc = ld;
    d.m = mi - c1; d.n = ni - c1; d.k = ib;
    d.alpha = -1.0; d.beta = 1.0;
    return true;
}

// Deferred left-block interchanges of the L1 kernel (a4.2).
// The columns of panel q need, in order, the interchanges of every later
// panel; no step of the factorization reads them again, so instead of moving
// up to 2 ib scattered rows of the whole left block after every panel (one
// 32-byte sector per 8-byte element) they are permuted once at the end.  With
// g the gather map of the later panels' interchanges (column y = x[g]), panels
// are processed right to left: g <- h_{q+1} o g, where h_{q+1} is the identity
// with panel q+1's swaps applied in order, then the rows [j_{q+1}, m) of
// panel q's columns are read (coalesced, cp.async) and written back permuted.
template <int NT>
__device__ __forceinline__ void left_swaps_core(double *__restrict__ gA, long ld, int mi, int K, int nb,
                                                const int *__restrict__ gip, int *g, int *h, double *buf,
                                                int cap) {
    const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
    for (int r = tid; r < mi; r += NT) g[r] = r;
    const int npan = (K + nb - 1) / nb;
    for (int q = npan - 2; q >= 0; --q) {
        const int js = (q + 1) * nb, ibn = imin(nb, K - js);
        for (int r = js + tid; r < mi; r += NT) h[r] = r;
        __syncthreads();
        if (tid == 0) {
            for (int t = 0; t < ibn; ++t) {
                const int p = gip[js + t] - 1;
                if (p != js + t) {
                    const int x = h[js + t];
                    h[js + t] = h[p];
                    h[p] = x;
                }
            }
        }
        __syncthreads();
        for (int r = js + tid; r < mi; r += NT) g[r] = h[g[r]];
        __syncthreads();
        const int rows = mi - js, c0 = q * nb;
        int W = cap / rows;
        W = W < 1 ? 1 : (W > nb ? nb : W);
        for (int cb = 0; cb < nb; cb += W) {
            const int w = imin(W, nb - cb);
            for (int c = warp; c < w; c += NT / 32) {
                const double *gc = gA + js + (size_t)(c0 + cb + c) * ld;
                for (int r = lane; r < rows; r += 32) cp_async8(buf + r + (size_t)c * rows, gc + r);
            }
            cp_async_commit();
            cp_async_wait<0>();
            __syncthreads();
            for (int c = warp; c < w; c += NT / 32) {
                double *gc = gA + js + (size_t)(c0 + cb + c) * ld;
                for (int r = lane; r < rows; r += 32) {
                    const int src = g[js + r] - js;
                    if (src != r) gc[r] = buf[src + (size_t)c * rows];
                }
            }
            __syncthreads();
        }
    }
}

__device__ __noinline__ void l1_left_swaps(double *__restrict__ gA, long ld, int mi, int K, int nb,
                                           const int *__restrict__ gip, double *smd, int region_doubles) {
    int *g = reinterpret_cast<int *>(smd);
    // past the two int maps (2 x 1024 x 4 B)
    left_swaps_core<L1_NT>(gA, ld, mi, K, nb, gip, g, g + L1_TALL_ROWS, smd + L1_TALL_ROWS,
                           region_doubles - L1_TALL_ROWS);
}

// ================================================================== L1
// One CTA per matrix, all iterations inside (matrices with m <= L1 rows).
// tall L1 panels (257..1024 rows)
__device__ __forceinline__ int l1_panel_tall(double *gP, long ld, int rows, int ib, int *piv,
                                          PanelWinSmem<L1_NT / 32, 32> &pws) {
    return rows <= 4 * L1_NT ? panel_win<L1_NT, 4, 8, 32>(gP, ld, rows, ib, piv, pws)
                             : panel_win<L1_NT, 8, 4, 32>(gP, ld, rows, ib, piv, pws);
}

// Matrices are taken largest first (LPT): `order` is the L1 list sorted by
// descending work (l1_key_kernel + the device size sort), `order_count` its
// length; without a sort the classify order is used.
// Panels of up to 256 rows are staged in shared memory and factored in
// registers (panel_regs); taller ones (<= 1024 rows) are factored in place in
// global memory by the windowed register panel (panel_win).
template <bool DMMA, bool TALL>
__global__ void __launch_bounds__(L1_NT, 3) lu_l1_kernel(GetrfArgs a, int *__restrict__ counters,
                                                         const int *__restrict__ bins, int nb,
                                                         int l1_region_doubles, int phase_timing,
                                                         const int *__restrict__ order,
                                                         const int *__restrict__ order_count, int defer) {
    extern __shared__ __align__(16) unsigned char l1_smem[];
    __shared__ PanelScratch sc;
    __shared__ __align__(16) PanelRegScratch<L1_NT / 32, 32> prs;
    __shared__ SwapPlan sp;
    __shared__ int piv_s[NBMAX];
    __shared__ int next_s;
    double *smd = reinterpret_cast<double *>(l1_smem);
    GemmSmem &gsm = *reinterpret_cast<GemmSmem *>(l1_smem);
    PanelWinSmem<L1_NT / 32, 32> &pws = *reinterpret_cast<PanelWinSmem<L1_NT / 32, 32> *>(l1_smem);
    const int tid = threadIdx.x;
    const int count = order ? *order_count : counters[CNT_BIN0 + BIN_L1];
    const int *list = order ? order : bins + (size_t)BIN_L1 * a.batch;
    while (true) {
        if (tid == 0) next_s = atomicAdd(&counters[CNT_L1_NEXT], 1);
        __syncthreads();
        const int t = next_s;
        __syncthreads();
        if (t >= count) break;
        const int i = list[t];
        const int mi = a.m[i], ni = a.n[i];
        const long ld = a.ld[i];
        double *gA = a.A[i];
        int *gip = a.ipiv[i];
        const int K = mi < ni ? mi : ni;
        int info = 0;
        unsigned long long *ph = reinterpret_cast<unsigned long long *>(counters + CNT_PHASE0);
        long long t0 = phase_timing ? clock64() : 0;
        for (int j = 0; j < K; j += nb) {
            const int ib = K - j < nb ? K - j : nb;
            const int rows = mi - j, c1 = j + ib;
            // ---- a4.1 panel, staged in shared memory (<= 256 rows) or in place
            double *gP = gA + j + (size_t)j * ld;
            const bool staged = !TALL || rows <= L1_MAX_ROWS;
            double *P = staged ? smd : gP;
            const int ldp = staged ? (rows | 1) : (int)ld;
            if (staged) {
                stage_block_async(P, ldp, gP, ld, rows, ib, tid, L1_NT);
                cp_async_commit();
                cp_async_wait<0>();
                __syncthreads();
            }
            if (phase_timing && tid == 0) { long long t1 = clock64(); atomicAdd(ph + 3, (unsigned long long)(t1 - t0)); t0 = t1; }
            const bool regs_panel = ib <= 32;
            int z;
            if (staged) {
                z = regs_panel ? panel_regs<L1_NT, 2, 32>(P, ldp, rows, ib, piv_s, prs, &sp, j)
                               : panel_getf2<L1_NT>(P, ldp, 0, rows, 0, ib, 0, ib, piv_s, sc);
            } else if (TALL && regs_panel) {
                z = l1_panel_tall(gP, ld, rows, ib, piv_s, pws);
                // the plan in absolute rows for the interchange pass
                if (tid < ib) sp.top_src[tid] = j + pws.plan.top_src[tid];
                if (tid < pws.plan.nbot) {
                    sp.bot_pos[tid] = j + pws.plan.bot_pos[tid];
                    sp.bot_src[tid] = j + pws.plan.bot_src[tid];
                }
                if (tid == 0) sp.nbot = pws.plan.nbot;
                __syncthreads();
            } else {
                z = panel_getf2<L1_NT>(P, ldp, 0, rows, 0, ib, 0, ib, piv_s, sc);
            }
            if (phase_timing && tid == 0) { long long t1 = clock64(); atomicAdd(ph + 4, (unsigned long long)(t1 - t0)); t0 = t1; }
            if (z && !info) info = j + z;
            // write the factored panel back; keep the strict lower triangle of
            // L11, packed by columns, past the union region for the U12 solve
            double *L11p = smd + l1_region_doubles;
            {
                const int lane = tid & 31, warp = tid >> 5;
                for (int c = warp; c < ib; c += L1_NT / 32) {
                    double *gc = gP + (size_t)c * ld;
                    const double *pc = P + (size_t)c * ldp;
                    if (staged)
                        for (int r = lane; r < rows; r += 32) gc[r] = pc[r];
                    double *lc = L11p + (c * (2 * ib - c - 1)) / 2 - (c + 1);
                    for (int r = c + 1 + lane; r < ib; r += 32) lc[r] = pc[r];
                }
            }
            if (tid < ib) {
                piv_s[tid] += j;                  // absolute row
                gip[j + tid] = piv_s[tid] + 1;
            }
            __syncthreads();
            if (phase_timing && tid == 0) { long long t1 = clock64(); atomicAdd(ph + 0, (unsigned long long)(t1 - t0)); t0 = t1; }
            // ---- a4.2 + a4.3 interchanges left / right, U12 solve
            if ((j > 0 && !defer) || c1 < ni) {
                double *top = smd;
                double *bot = top + nb * (SW_COLS + 1);
                if (!regs_panel) {  // panel_regs already emitted the plan
                    plan_swaps_from(piv_s, j, ib, sp);
                    __syncthreads();
                }
                unsigned long long *phs = phase_timing ? ph : nullptr;
                if (phase_timing && tid == 0) { long long t1 = clock64(); atomicAdd(ph + 1, (unsigned long long)(t1 - t0)); t0 = t1; }
                // left block [0, j) (unless deferred) and right block [c1, n)
                // as one virtual range
                const int jl = defer ? 0 : j;
                const int vtot = jl + (ni - c1);
                for (int vb = 0; vb < vtot; vb += SW_COLS)
                    swap_chunk(gA, ld, j, ib, vb, imin(SW_COLS, vtot - vb), jl, c1 - jl, c1, sp, L11p, 0, top, bot,
                               phs);
            }
            if (phase_timing && tid == 0) t0 = clock64();  // chunk phases were accounted in slots 5..7
            // ---- a4.4 trailing update through the pipelined GEMM core
            GemmDesc d0;
            if (trailing_desc(gA, ld, mi, ni, j, nb, d0)) {
                const int ntm = (d0.m + GBM - 1) / GBM, ntiles = ntm * ((d0.n + GBN - 1) / GBN);
                int tt = 0;
                auto next = [&](GemmDesc &d, int &r0, int &cc0) -> bool {
                    if (tt >= ntiles) return false;
                    d = d0;
                    r0 = (tt % ntm) * GBM;
                    cc0 = (tt / ntm) * GBN;
                    ++tt;
                    return true;
                };
                gemm_tile_stream<DMMA, decltype(next), false, false, false>(next, gsm);
            }
            __syncthreads();
            if (phase_timing && tid == 0) { long long t1 = clock64(); atomicAdd(ph + 2, (unsigned long long)(t1 - t0)); t0 = t1; }
        }
        if (defer && K > nb) l1_left_swaps(gA, ld, mi, K, nb, gip, smd, l1_region_doubles);
        if (tid == 0) a.info[i] = info;
    }
}

// ================================================================== L2
__global__ void __launch_bounds__(P_NT) panel_kernel(GetrfArgs a, const int *__restrict__ counters,
                                                     const int *__restrict__ bins, int j, int nb, int smem_rows) {
    extern __shared__ __align__(16) double sp_panel[];
    __shared__ PanelScratch sc;
    __shared__ __align__(16) PanelRegScratch<P_NT / 32, 32> prs;
    __shared__ int piv_s[NBMAX];
    const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
    constexpr int NW = P_NT / 32;
    const int count = counters[CNT_BIN0 + BIN_L];
    const int *list = bins + (size_t)BIN_L * a.batch;
    for (int t = blockIdx.x; t < count; t += gridDim.x) {
        const int i = list[t];
        const int mi = a.m[i], ni = a.n[i], ld = a.ld[i];
        const int K = mi < ni ? mi : ni;
        if (j >= K) continue;  // DCWI: no work
        const int ib = K - j < nb ? K - j : nb;
        const int rows = mi - j;
        double *gP = a.A[i] + j + (size_t)j * ld;
        double *P;
        int ldp;
        const bool staged = rows <= smem_rows;
        if (staged) {
            ldp = rows | 1;
            P = sp_panel;
            stage_block_async(P, ldp, gP, ld, rows, ib, tid, P_NT);
            cp_async_commit();
            cp_async_wait<0>();
            __syncthreads();
        } else {
            P = gP;
            ldp = ld;
        }
        int z = (staged && ib <= 32 && rows <= 2 * P_NT)
                    ? panel_regs<P_NT, 2, 32>(P, ldp, rows, ib, piv_s, prs)
                    : panel_getf2<P_NT>(P, ldp, 0, rows, 0, ib, 0, ib, piv_s, sc);
        if (staged) {
            for (int c = warp; c < ib; c += NW)
                for (int r = lane; r < rows; r += 32) gP[r + (size_t)c * ld] = P[r + c * ldp];
        }
        if (tid < ib) a.ipiv[i][j + tid] = j + piv_s[tid] + 1;
        if (tid == 0 && z && a.info[i] == 0) a.info[i] = j + z;
        __syncthreads();
    }
}

// Windowed register panel straight on global memory (panel_win.cuh): rows
// <= 2048 in registers (RPT = 2, 4, 8 with window 16, 8, 4), 2 CTAs / SM, by
// 256 threads; taller panels (the few-large regime) by
// 512 threads (<= 4096 rows, window 4) or 1024 threads (<= 8192 rows,
// window 2); beyond that the global-memory panel_getf2.
constexpr int PW_NT = 256;
constexpr int PW_MAX_ROWS = 8192;
template <int NT>
__global__ void __launch_bounds__(NT, NT <= 256 ? 2 : 1) panel_win_kernel(GetrfArgs a, const int *__restrict__ counters,
                                                                         const int *__restrict__ bins, int j, int nb,
                                                                         SwapPlan *__restrict__ plans, int *queue,
                                                                         int *pqueue) {
    extern __shared__ __align__(16) double pw_smem[];
    PanelWinSmem<NT / 32> &sm = *reinterpret_cast<PanelWinSmem<NT / 32> *>(pw_smem);
    __shared__ PanelScratch sc;
    __shared__ int piv_s[NBMAX];
    const int tid = threadIdx.x;
    __shared__ int item_s;
    const int count = counters[CNT_BIN0 + BIN_L];
    const int *list = bins + (size_t)BIN_L * a.batch;
    if (blockIdx.x == 0 && tid == 0) *queue = 0;  // the strip kernel's work queue (stream-ordered)
    for (;;) {
        // dynamic queue over the LPT-ordered list (reset by the kernel that follows)
        if (tid == 0) item_s = atomicAdd(pqueue, 1);
        __syncthreads();
        const int t = item_s;
        __syncthreads();
        if (t >= count) break;
        const int i = list[t];
        const int mi = a.m[i], ni = a.n[i], ld = a.ld[i];
        const int K = mi < ni ? mi : ni;
        if (j >= K) continue;  // DCWI: no work
        const int ib = K - j < nb ? K - j : nb;
        const int rows = mi - j;
        double *gP = a.A[i] + j + (size_t)j * ld;
        int z;
        bool planned = true;
        if (NT == 256 && rows <= 2 * NT) z = panel_win<NT, 2, 16>(gP, ld, rows, ib, piv_s, sm);
        else if (NT == 256 && rows <= 4 * NT) z = panel_win<NT, 4, 8>(gP, ld, rows, ib, piv_s, sm);
        else if (NT <= 512 && rows <= 8 * NT) z = panel_win<NT, 8, 4>(gP, ld, rows, ib, piv_s, sm);
        else if (NT == 1024 && rows <= 8 * NT) z = panel_win<NT, 8, 2>(gP, ld, rows, ib, piv_s, sm);
        else {
            z = panel_getf2<NT>(gP, ld, 0, rows, 0, ib, 0, ib, piv_s, sc);
            planned = false;
        }
        if (planned) {
            // the interchange plan for the strip kernel (absolute rows)
            SwapPlan &g = plans[t];
            if (tid < ib) g.top_src[tid] = j + sm.plan.top_src[tid];
            if (tid < sm.plan.nbot) {
                g.bot_pos[tid] = j + sm.plan.bot_pos[tid];
                g.bot_src[tid] = j + sm.plan.bot_src[tid];
            }
            if (tid == 0) g.nbot = sm.plan.nbot;
        }
        if (tid < ib) a.ipiv[i][j + tid] = j + piv_s[tid] + 1;
        if (tid == 0 && z && a.info[i] == 0) a.info[i] = j + z;
        __syncthreads();
    }
}

// the windowed panel for the tallest panel of the launch
static void launch_panel_win(int max_rows, int grid, const GetrfArgs &a, int *counters, const int *bins, int j,
                             int nb, SwapPlan *plans, int *queue, cudaStream_t s) {
    int *pq = counters + CNT_PANELQ;
    if (max_rows <= 8 * 256) {
        panel_win_kernel<256><<<grid, 256, sizeof(PanelWinSmem<8>), s>>>(a, counters, bins, j, nb, plans, queue, pq);
    } else if (max_rows <= 8 * 512) {
        const int g = grid < num_sms() ? grid : num_sms();
        panel_win_kernel<512><<<g, 512, sizeof(PanelWinSmem<16>), s>>>(a, counters, bins, j, nb, plans, queue, pq);
    } else {
        const int g = grid < num_sms() ? grid : num_sms();
        panel_win_kernel<1024><<<g, 1024, sizeof(PanelWinSmem<32>), s>>>(a, counters, bins, j, nb, plans, queue, pq);
    }
}

// Fused step a4.2 + a4.3 + a4.4 of the grid-wide tier, one work item per
// (tier-L slot, 64-column strip of the virtual range [0, n - ib)): gather the
// moved rows of the strip (plan from the panel kernel), solve the U12 part with
// the unit L11, scatter, then stream the trailing GEMM down the strip,
// C(c1:m, strip) -= L21 U12(:, strip).  The interchanged rows are re-read by
// the GEMM straight from L2, and every strip is owned by exactly one CTA, so
// no other CTA can observe a half-swapped column.  Items come from a dynamic
// queue (reset by the panel kernel).
constexpr int ST_COLS = GBN;
constexpr int SPLIT_BATCH = 32;  // split_strip = 2: batches up to this many matrices
static_assert(sizeof(SwapPlan) <= SWAP_PLAN_BYTES, "plan slot");
template <bool DMMA>
__global__ void __launch_bounds__(G_NT, 3) strip_kernel(GetrfArgs a, int *__restrict__ counters,
                                                        const int *__restrict__ bins,
                                                        const SwapPlan *__restrict__ plans, int *queue, int j,
                                                        int nb, int chunks_per, unsigned long long *ph, int defer,
                                                        int J, int cmax, int do_gemm = 1) {
    extern __shared__ __align__(16) double st_smem[];
    GemmSmem &gsm = *reinterpret_cast<GemmSmem *>(st_smem);
    const int ldl = nb + 1;
    // nb <= 32: the solved U12 rows (top) ARE the GEMM's resident B operand
    // (gsm.Bs: 2 x 16 rows of stride GPAD), and L11 / bot sit in the C
    // stage (dead during the interchange + TRSM, filled only by the GEMM
    // tiles afterwards); else the original layout
    const bool bres = DMMA && nb <= 2 * GBK;
    double *top = bres ? &gsm.Bs[0][0][0] : st_smem + nb * ldl;
    double *L11 = bres ? &gsm.Cs[0][0] : st_smem;
    double *bot = bres ? L11 + nb * ldl : top + nb * GPAD;
    __shared__ SwapPlan sp;
    __shared__ int item_s;
    const int tid = threadIdx.x;
    const int count = counters[CNT_BIN0 + BIN_L];
    const int *list = bins + (size_t)BIN_L * a.batch;
    const long long total = (long long)count * chunks_per;
    int last_slot = -1;
    long long t0 = (ph && tid == 0) ? clock64() : 0;
    if (blockIdx.x == 0 && tid == 0) counters[CNT_PANELQ] = 0;  // the next panel launch's queue (stream-ordered)
#define ST_PHASE(k)                                                           \
    if (ph && tid == 0) {                                                     \
        long long t1 = clock64();                                             \
        atomicAdd(ph + (k), (unsigned long long)(t1 - t0));                   \
        t0 = t1;                                                              \
    }
    for (;;) {
        ST_PHASE(3)  // the tail of empty items
        if (tid == 0) item_s = atomicAdd(queue, 1);
        __syncthreads();
        const long long w = item_s;
        __syncthreads();  // every thread has read item_s before thread 0 takes the next item
        if (w >= total) break;
        const int slot = (int)(w / chunks_per), q = (int)(w - (long long)slot * chunks_per);
        const int i = list[slot];
        const int mi = a.m[i], ni = a.n[i], ld = a.ld[i];
        const int K = mi < ni ? mi : ni;
        if (j >= K) continue;
        const int ib = K - j < nb ? K - j : nb;
        const int c1 = j + ib;
        // virtual columns v in [lb, j + nright): v < j is left-block column v
        // (interchanges only), v >= j is column v + ib of the right block
        // [c1, ce) (interchanges + U12 solve + GEMM).  One level: lb = 0 (eager)
        // or j (left block deferred to left_swaps_kernel), ce = n.  Two-level
        // (J >= 0): the inner step works inside the outer block [J, cmax):
        // lb = J, ce = min(n, cmax); columns outside it get the outer block's
        // interchanges later (outer_swap_trsm_kernel / left_swaps_kernel).
        const int lb = J >= 0 ? J : (defer ? j : 0);
        const int ce = J >= 0 ? imin(imin(ni, cmax), K) : ni;  // an outer block ends at min(J + nbo, K)
        const int nright = ce > c1 ? ce - c1 : 0;
        const int vtot = (j - lb) + nright, vb = q * ST_COLS;
        if (vb >= vtot) continue;
        double *gA = a.A[i];
        if (slot != last_slot) {
            const int *src = reinterpret_cast<const int *>(plans + slot);
            int *dst = reinterpret_cast<int *>(&sp);
            for (int e = tid; e < (int)(sizeof(SwapPlan) / sizeof(int)); e += G_NT) dst[e] = src[e];
            last_slot = slot;
        }
        load_L11_async(L11, ldl, gA, ld, j, ib);
        cp_async_commit();
        __syncthreads();
        ST_PHASE(0)
        const int W = imin(ST_COLS, vtot - vb);
        const int v0 = lb + vb;  // first virtual column of the strip
        // row stride GPAD: top doubles as the GEMM's resident B stage
        swap_chunk<ST_COLS, GPAD>(gA, ld, j, ib, v0, W, j, ib, c1, sp, L11, ldl, top, bot, ph);
        if (ph && tid == 0) t0 = clock64();
        // trailing GEMM on the strip's right-of-panel columns
        const int cbeg = (v0 > j ? v0 : j) + ib, cend = v0 + W + ib;
        if (do_gemm && cbeg < cend && c1 < mi) {
            GemmDesc d0;
            d0.A = gA + c1 + (size_t)j * ld; d0.lda = ld; d0.ta = 0;
            d0.B = gA + j + (size_t)cbeg * ld; d0.ldb = ld; d0.tb = 0;
            d0.C = gA + c1 + (size_t)cbeg * ld; d0.ldc = ld;
            d0.m = mi - c1; d0.n = cend - cbeg; d0.k = ib;
            d0.alpha = -1.0; d0.beta = 1.0;
            const int ntm = (d0.m + GBM - 1) / GBM;
            int tt = 0;
            auto next = [&](GemmDesc &d, int &r0, int &cc0) -> bool {
                if (tt >= ntm) return false;
                d = d0;
                r0 = tt * GBM;
                cc0 = 0;
                ++tt;
                return true;
            };
            if (bres && v0 >= j) {  // the GEMM's columns start at top's column 0
                // B rows >= ib of the resident operand must be zero (A is
                // zero-filled there, but stale shared memory may hold NaNs)
                if (ib < 2 * GBK)
                    for (int e = tid; e < (2 * GBK - ib) * GPAD; e += G_NT) top[ib * GPAD + e] = 0.0;
                __syncthreads();
                gemm_tile_stream<DMMA, decltype(next), false, true>(next, gsm);
            } else {
                gemm_tile_stream<DMMA>(next, gsm);
            }
            __syncthreads();
            ST_PHASE(2)
        }
    }
#undef ST_PHASE
}

// The deferred left-block interchanges of the grid-wide tier: one CTA per
// tier-L matrix (dynamic queue), after the last panel (left_swaps_core).
constexpr int LSW_NT = 256;
constexpr int LSW_BUF = 6144;  // doubles of column buffer (48 KB), at least one full column (max_m)
static int lsw_buf_doubles(int max_m) { return max_m > LSW_BUF ? ((max_m + 1) & ~1) : LSW_BUF; }
__global__ void __launch_bounds__(LSW_NT) left_swaps_kernel(GetrfArgs a, const int *__restrict__ counters,
                                                            const int *__restrict__ bins, int nb, int maps,
                                                            int bufd, int *queue) {
    extern __shared__ __align__(16) double lsw_smem[];
    __shared__ int item_s;
    double *buf = lsw_smem;
    int *g = reinterpret_cast<int *>(lsw_smem + bufd);
    int *h = g + maps;
    const int count = counters[CNT_BIN0 + BIN_L];
    const int *list = bins + (size_t)BIN_L * a.batch;
    for (;;) {
        if (threadIdx.x == 0) item_s = atomicAdd(queue, 1);
        __syncthreads();
        const int t = item_s;
        __syncthreads();
        if (t >= count) break;
        const int i = list[t];
        const int mi = a.m[i], ni = a.n[i];
        const int K = mi < ni ? mi : ni;
        if (K > nb) left_swaps_core<LSW_NT>(a.A[i], a.ld[i], mi, K, nb, a.ipiv[i], g, h, buf, bufd);
    }
}


// ================================================================== two-level grid tier
// Outer blocks of NBo (<= NB_OUTER_MAX) columns, each factored by NBo / nb
// inner panel steps confined to the block (panel_win_kernel + strip_kernel
// with J >= 0), then ONE update of the rest of the matrix per outer block
// (P:L106's blocked right-looking LU with panel width NBo, the panel itself
// blocked): the composed interchanges of the NBo pivots + U12 <- L11^-1 A12
// (outer_swap_trsm_kernel) and A22 -= L21 U12 with K = NBo on the 128 x 128
// DMMA core (xgemm).  The trailing matrix is streamed once per NBo columns
// instead of once per nb: arithmetic intensity NBo / 8 flop/B instead of
// nb / 8 (SURVEY §7 hard part 1).

// one warp per tier-L slot composes the outer block's interchanges
// ipiv[J .. J + ibo) into a plan (absolute rows); block 0 resets the queue
// of outer_swap_trsm_kernel (stream-ordered)
constexpr int OP_NT = 256;
__global__ void __launch_bounds__(OP_NT) outer_plan_kernel(GetrfArgs a, const int *__restrict__ counters,
                                                           const int *__restrict__ bins, int J, int NBo,
                                                           OuterPlan *__restrict__ plans, int *queue) {
    __shared__ OuterPlan sp[OP_NT / 32];
    const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
    if (blockIdx.x == 0 && threadIdx.x == 0) *queue = 0;
    const int count = counters[CNT_BIN0 + BIN_L];
    const int *list = bins + (size_t)BIN_L * a.batch;
    OuterPlan &p = sp[warp];
    for (int t = blockIdx.x * (OP_NT / 32) + warp; t < count; t += gridDim.x * (OP_NT / 32)) {
        const int i = list[t];
        const int mi = a.m[i], ni = a.n[i];
        const int K = mi < ni ? mi : ni;
        if (J >= K) continue;
        const int ibo = imin(NBo, K - J);
        if (J + ibo >= ni) continue;  // no columns right of the block
        const int *ip = a.ipiv[i];
        for (int q = lane; q < ibo; q += 32) p.piv[q] = ip[J + q] - 1;
        __syncwarp();
        plan_swaps_core(J, ibo, p);
        __syncwarp();
        OuterPlan &g = plans[t];
        for (int q = lane; q < ibo; q += 32) g.top_src[q] = p.top_src[q];
        const int nbot = p.nbot;
        for (int q = lane; q < nbot; q += 32) {
            g.bot_pos[q] = p.bot_pos[q];
            g.bot_src[q] = p.bot_src[q];
        }
        if (lane == 0) g.nbot = nbot;
        __syncwarp();
    }
}

// Right of outer block [J, J + ibo): per (tier-L matrix, OS_COLS-column
// strip), over a DENSE item space (per-matrix strip counts prefix-summed on
// the device; each persistent CTA walks a contiguous range, so consecutive
// strips of one matrix share the CTA and its L11):
//   0. on a new matrix: the unit-lower L11 (ibo x ibo) staged in shared memory
//      once, and the block's composed interchange plan (outer_plan_kernel);
//   1. one thread per moved row: the ibo rows that end in [J, J + ibo) are
//      gathered into shared memory (cp.async), the <= ibo rows pushed below
//      the block are read into registers and -- after every read of the
//      strip -- written to their new rows;
//   2. U12 <- L11^-1 U12 in 32-row blocks: the diagonal block by a warp-wide
//      substitution (lane = row, 8 columns per warp, the solved entry
//      broadcast by shuffle), the rows below it by a rank-32 DMMA update
//      (m8n8k4, both operands in shared memory);
//   3. U12 back to rows [J, J + ibo), one thread per row (coalesced).
// Two shapes: 64-column strips with L11 in a padded square (1 CTA / SM,
// 206 KB), or 32-column strips with L11's strict lower triangle packed by
// columns (2 CTAs / SM, 101 KB) -- tuning outer_cols.
constexpr int OS_NT = 256, OS_LDL = 136;
constexpr int OS_LPACK = NB_OUTER_MAX * (NB_OUTER_MAX - 1) / 2;
template <int COLS>
struct OsCfg {
    static constexpr bool PACK = COLS <= 32;
    static constexpr int TLD = COLS + 1;
    static constexpr size_t SMEM =
        (size_t)(NB_OUTER_MAX * TLD + (PACK ? OS_LPACK : NB_OUTER_MAX * OS_LDL)) * sizeof(double);
    // L11(r, s), r > s
    __device__ static __forceinline__ int lidx(int r, int s) {
        return PACK ? s * (2 * NB_OUTER_MAX - 1 - s) / 2 + (r - s - 1) : s * OS_LDL + r;
    }
};

template <int COLS>
struct OuterStrips {
    GetrfArgs a;
    const int *list;
    int J, NBo;
    __device__ int units(int slot) const {
        const int i = list[slot];
        const int mi = a.m[i], ni = a.n[i];
        const int K = mi < ni ? mi : ni;
        if (J >= K) return 0;
        const int c1 = J + imin(NBo, K - J);
        return c1 < ni ? (ni - c1 + COLS - 1) / COLS : 0;
    }
};

template <int COLS>
__global__ void __launch_bounds__(OS_NT, COLS <= 32 ? 2 : 1) outer_swap_trsm_kernel(
    GetrfArgs a, const int *__restrict__ counters, const int *__restrict__ bins, const OuterPlan *__restrict__ plans,
    const int *__restrict__ off, int J, int NBo) {
    using Cfg = OsCfg<COLS>;
    constexpr int TLD = Cfg::TLD;
    extern __shared__ __align__(16) double os_smem[];
    double *top = os_smem;                       // U12 rows: top[t * TLD + c]
    double *Ls = top + NB_OUTER_MAX * TLD;       // L11 strict lower: Ls[Cfg::lidx(r, s)]
    __shared__ OuterPlan sp;
    const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
    const int g = lane >> 2, t4 = lane & 3;
    constexpr int NWS = OS_NT / 32;
    constexpr int CPW = COLS / NWS;   // diagonal-solve columns per warp
    const int count = counters[CNT_BIN0 + BIN_L];
    const int *list = bins + (size_t)BIN_L * a.batch;
    int last_slot = -1;
    auto strip = [&](int slot, int q) {
        const int i = list[slot];
        const int mi = a.m[i], ni = a.n[i];
        const int K = mi < ni ? mi : ni;
        const int ibo = imin(NBo, K - J), c1 = J + ibo;
        const int cb = c1 + q * COLS;
        const int W = imin(COLS, ni - cb);
        const long ld = a.ld[i];
        double *gA = a.A[i];
        if (slot != last_slot) {
            __syncthreads();
            const int *src = reinterpret_cast<const int *>(plans + slot);
            int *dst = reinterpret_cast<int *>(&sp);
            for (int e = tid; e < (int)(sizeof(OuterPlan) / sizeof(int)); e += OS_NT) dst[e] = src[e];
            // strict lower part of L11, column by column (lanes over rows)
            for (int sc = warp; sc < ibo - 1; sc += NWS) {
                const double *gl = gA + J + (size_t)(J + sc) * ld;
                for (int r = sc + 1 + lane; r < ibo; r += 32) cp_async8(&Ls[Cfg::lidx(r, sc)], gl + r);
            }
            last_slot = slot;
        }
        __syncthreads();
        const int nbot = sp.nbot;
        // ---- 1. gather: threads [0, 128) the top rows, [128, 256) the rows pushed down
        const double *gcb = gA + (size_t)cb * ld;
        double bv[COLS];
        if (tid < NB_OUTER_MAX) {
            if (tid < ibo) {
                const double *src = gcb + sp.top_src[tid];
                double *dst = top + tid * TLD;
#pragma unroll 8
                for (int c = 0; c < W; ++c) cp_async8(dst + c, src + (size_t)c * ld);
            }
        } else {
            const int b = tid - NB_OUTER_MAX;
            if (b < nbot) {
                const double *src = gcb + sp.bot_src[b];
#pragma unroll
                for (int c = 0; c < COLS; ++c) bv[c] = c < W ? src[(size_t)c * ld] : 0.0;
            }
        }
        cp_async_commit();
        cp_async_wait<0>();
        __syncthreads();
        if (tid >= NB_OUTER_MAX) {
            const int b = tid - NB_OUTER_MAX;
            if (b < nbot) {
                double *dst = gA + (size_t)cb * ld + sp.bot_pos[b];
#pragma unroll
                for (int c = 0; c < COLS; ++c)
                    if (c < W) dst[(size_t)c * ld] = bv[c];
            }
        }
        // ---- 2. U12 <- L11^-1 U12, 32-row blocks
        for (int d0 = 0; d0 < ibo; d0 += 32) {
            const int bw = imin(32, ibo - d0);
            const int below = ibo - d0 - bw;
            {   // diagonal block: warp w solves columns [CPW w, CPW w + CPW), lane = row
                const int c0 = warp * CPW;
                double x[CPW];
#pragma unroll
                for (int c = 0; c < CPW; ++c) x[c] = (lane < bw && c0 + c < W) ? top[(d0 + lane) * TLD + c0 + c] : 0.0;
                for (int sc = 0; sc < bw - 1; ++sc) {
                    const double l = (lane > sc && lane < bw) ? Ls[Cfg::lidx(d0 + lane, d0 + sc)] : 0.0;
#pragma unroll
                    for (int c = 0; c < CPW; ++c) x[c] = fma(-l, __shfl_sync(FULL, x[c], sc), x[c]);
                }
                if (lane < bw)
#pragma unroll
                    for (int c = 0; c < CPW; ++c)
                        if (c0 + c < W) top[(d0 + lane) * TLD + c0 + c] = x[c];
            }
            __syncthreads();
            if (below > 0) {   // rows below: 32 x 32 output tiles per warp (DMMA)
                const int tiles_m = (below + 31) / 32, tiles = tiles_m * (COLS / 32);
                for (int tt = warp; tt < tiles; tt += NWS) {
                    const int rb = (tt % tiles_m) * 32, cbt = (tt / tiles_m) * 32;
                    double acc[4][4][2];
#pragma unroll
                    for (int mi = 0; mi < 4; ++mi)
#pragma unroll
                        for (int n8 = 0; n8 < 4; ++n8) { acc[mi][n8][0] = 0.0; acc[mi][n8][1] = 0.0; }
#pragma unroll
                    for (int ks = 0; ks < 32; ks += 4) {
                        const int sc = ks + t4;
                        double av[4], bb[4];
#pragma unroll
                        for (int mi = 0; mi < 4; ++mi) {
                            const int r = rb + 8 * mi + g;   // row under the diagonal block
                            av[mi] = (sc < bw && r < below) ? Ls[Cfg::lidx(d0 + bw + r, d0 + sc)] : 0.0;
                        }
#pragma unroll
                        for (int n8 = 0; n8 < 4; ++n8) {
                            const int c = cbt + 8 * n8 + g;
                            bb[n8] = (sc < bw && c < W) ? top[(d0 + sc) * TLD + c] : 0.0;
                        }
#pragma unroll
                        for (int mi = 0; mi < 4; ++mi)
#pragma unroll
                            for (int n8 = 0; n8 < 4; ++n8) dmma_8x8x4(acc[mi][n8][0], acc[mi][n8][1], av[mi], bb[n8]);
                    }
#pragma unroll
                    for (int mi = 0; mi < 4; ++mi) {
                        const int r = rb + 8 * mi + g;
                        if (r >= below) continue;
                        double *row = top + (size_t)(d0 + bw + r) * TLD;
#pragma unroll
                        for (int n8 = 0; n8 < 4; ++n8) {
                            const int c = cbt + 8 * n8 + 2 * t4;
                            if (c < W) row[c] -= acc[mi][n8][0];
                            if (c + 1 < W) row[c + 1] -= acc[mi][n8][1];
                        }
                    }
                }
            }
            __syncthreads();
        }
        // ---- 3. U12 back to rows [J, J + ibo), one thread per row
        if (tid < ibo) {
            double *dst = gA + J + tid + (size_t)cb * ld;
            const double *src = top + tid * TLD;
#pragma unroll 8
            for (int c = 0; c < W; ++c) dst[(size_t)c * ld] = src[c];
        }
    };
    walk_units(SlotList{nullptr, nullptr, 0}, count, off, strip);
}

// A22 -= L21 U12 of outer block [J, J + ibo) for every tier-L matrix (K = ibo)
struct OuterTrailProb {
    GetrfArgs a;
    const int *list;
    int J, NBo;
    __device__ bool get(int slot, GemmDesc &d) const {
        const int i = list[slot];
        const int mi = a.m[i], ni = a.n[i];
        const int K = mi < ni ? mi : ni;
        d.m = 0; d.n = 0; d.k = 0;
        if (J >= K) return false;
        const int ibo = imin(NBo, K - J), c1 = J + ibo;
        if (c1 >= mi || c1 >= ni) return false;
        const long ld = a.ld[i];
        double *A = a.A[i];
        d.A = A + c1 + (size_t)J * ld; d.lda = ld; d.ta = 0;
        d.B = A + J + (size_t)c1 * ld; d.ldb = ld; d.tb = 0;
        d.C = A + c1 + (size_t)c1 * ld; d.ldc = ld;
        d.m = mi - c1; d.n = ni - c1; d.k = ibo;
        d.alpha = -1.0; d.beta = 1.0;
        return true;
    }
};

static size_t strip_smem_bytes(int nb) {
    size_t sw = (size_t)(nb * (nb + 1) + 2 * nb * GPAD) * sizeof(double);
    size_t m = sw > GEMM_SMEM ? sw : GEMM_SMEM;
    return (m + 15) & ~size_t(15);
}

// Work item = (tier-L slot, column chunk) over the virtual column range
// [0, n - ib): virtual v < j is column v (interchanges only), v >= j is column
// v + ib (interchanges + forward substitution with the unit L11).  Each CTA
// takes a CONTIGUOUS run of items, so consecutive items share a matrix and
// the interchange plan and L11 are built once per (CTA, matrix).
__global__ void __launch_bounds__(SW_NT) swap_trsm_kernel(GetrfArgs a, const int *__restrict__ counters,
                                                          const int *__restrict__ bins, int j, int nb,
                                                          int chunks_per) {
    extern __shared__ __align__(16) double sw_smem[];
    const int ldl = nb + 1;
    double *L11 = sw_smem;
    double *top = L11 + nb * ldl;
    double *bot = top + nb * (SW_COLS + 1);
    __shared__ SwapPlan sp;
    const int count = counters[CNT_BIN0 + BIN_L];
    const int *list = bins + (size_t)BIN_L * a.batch;
    const long long total = (long long)count * chunks_per;
    const long long w0 = total * blockIdx.x / gridDim.x, w1 = total * (blockIdx.x + 1) / gridDim.x;
    int last_i = -1;
    for (long long w = w0; w < w1; ++w) {
        const int slot = (int)(w / chunks_per), q = (int)(w - (long long)slot * chunks_per);
        const int i = list[slot];
        const int mi = a.m[i], ni = a.n[i], ld = a.ld[i];
        const int K = mi < ni ? mi : ni;
        if (j >= K) continue;
        const int ib = K - j < nb ? K - j : nb;
        const int c1 = j + ib;
        const int vtot = ni - ib, vb = q * SW_COLS;
        if (vb >= vtot) continue;
        double *gA = a.A[i];
        if (i != last_i) {
            __syncthreads();
            load_L11_async(L11, ldl, gA, ld, j, ib);
            cp_async_commit();
            plan_swaps(a.ipiv[i], j, ib, sp);
            last_i = i;
            __syncthreads();
        }
        swap_chunk(gA, ld, j, ib, vb, imin(SW_COLS, vtot - vb), j, ib, c1, sp, L11, ldl, top, bot);
    }
}

struct TrailingProb {
    GetrfArgs a;
    const int *list;
    int j, nb;
    __device__ bool get(int slot, GemmDesc &d) const {
        const int i = list[slot];
        return trailing_desc(a.A[i], a.ld[i], a.m[i], a.n[i], j, nb, d);
    }
};
template <>
struct gemm_creg_ok<TrailingProb> { static constexpr bool value = false; };  // measured: staged C is faster

// Few-large batches (tuning split_strip): the inner step's trailing update
// inside the outer block, C(c1:m, c1:ce) -= L21 U12, as its own grid-wide
// GEMM over 64 x 64 tiles.  The fused strip kernel streams a strip's whole
// column range in ONE CTA, so a batch of one or a few large matrices runs
// its inner steps on one or two CTAs; here every row tile is its own CTA.
struct InnerTrailProb {
    GetrfArgs a;
    const int *list;
    int j, nb, J, cmax;
    __device__ bool get(int slot, GemmDesc &d) const {
        const int i = list[slot];
        const int mi = a.m[i], ni = a.n[i];
        const int K = mi < ni ? mi : ni;
        d.m = 0; d.n = 0; d.k = 0;
        if (j >= K) return false;
        const int ib = K - j < nb ? K - j : nb;
        const int c1 = j + ib;
        const int ce = imin(imin(ni, cmax), K);
        if (c1 >= mi || c1 >= ce) return false;
        const long ld = a.ld[i];
        double *A = a.A[i];
        d.A = A + c1 + (size_t)j * ld; d.lda = ld; d.ta = 0;
        d.B = A + j + (size_t)c1 * ld; d.ldb = ld; d.tb = 0;
        d.C = A + c1 + (size_t)c1 * ld; d.ldc = ld;
        d.m = mi - c1; d.n = ce - c1; d.k = ib;
        d.alpha = -1.0; d.beta = 1.0;
        return true;
    }
};
template <>
struct gemm_creg_ok<InnerTrailProb> { static constexpr bool value = false; };


static int clamp_nb(int nb) { return nb < 1 ? 1 : (nb > NBMAX ? NBMAX : nb); }

// L1 shared memory: a union region (panel | swap buffers | GEMM stages) plus
// the packed L11 behind it.
static size_t l1_region_bytes(int nb) {
    size_t panel = (size_t)(L1_MAX_ROWS | 1) * nb * sizeof(double);
    size_t swap = (size_t)(2 * nb * (SW_COLS + 1)) * sizeof(double);
    size_t m = panel > swap ? panel : swap;
    m = m > GEMM_SMEM ? m : GEMM_SMEM;
    return (m + 15) & ~size_t(15);
}

// LPT key of a matrix of bin `bin`: 32 + cube root of its m n min(m,n) (>= 32,
// so the bucketed size sort puts every matrix of the bin before the zero keys
// of the rest)
__global__ void l1_key_kernel(GetrfArgs a, const int *__restrict__ counters, const int *__restrict__ bins,
                              int *__restrict__ key, int bin = BIN_L1) {
    const int count = counters[CNT_BIN0 + bin];
    const int *list = bins + (size_t)bin * a.batch;
    for (int t = blockIdx.x * blockDim.x + threadIdx.x; t < count; t += gridDim.x * blockDim.x) {
        const int i = list[t];
        const double m = a.m[i], n = a.n[i];
        key[i] = 32 + (int)cbrt(m * n * (m < n ? m : n));
    }
}

void launch_lu_l1(const GetrfArgs &a, int *counters, const int *bins, int *keys, int *sort_ws, cudaStream_t s) {
    const int nb = clamp_nb(tuning().nb);
    const size_t region = l1_region_bytes(nb);
    const size_t smem = region + (size_t)(nb * (nb - 1) / 2 + 2) * sizeof(double);
    smem_optin(lu_l1_kernel<true, false>, smem);
    smem_optin(lu_l1_kernel<false, false>, smem);
    smem_optin(lu_l1_kernel<true, true>, smem);
    smem_optin(lu_l1_kernel<false, true>, smem);
    int per_sm = tuning().l1_ctas_per_sm;
    if (per_sm < 1 || per_sm > 3) per_sm = 3;
    int grid = num_sms() * per_sm;
    if (grid > a.batch) grid = a.batch;
    const int rd = (int)(region / sizeof(double)), pt = tuning().phase_timing, df = tuning().defer;
    const bool dm = tuning().l1_dmma;  // default: DMMA (measured faster once the variant stopped spilling)
    // one launch per bin: matrices of 257..l1_rows rows (BIN_L1T) by the
    // tall-panel variant (windowed panels in place), the rest by the staged-
    // panel variant, which needs fewer registers; each walks its bin LPT first
    auto one = [&](int bin, bool tall) {
        const int *order = nullptr, *order_count = nullptr;
        if (keys && sort_ws) {
            cudaMemsetAsync(keys, 0, (size_t)a.batch * sizeof(int), s);
            {
                KScope k(K_MISC, s);
                int g = (a.batch + 255) / 256;
                l1_key_kernel<<<g < 1024 ? g : 1024, 256, 0, s>>>(a, counters, bins, keys, bin);
            }
            launch_size_sort(keys, a.batch, sort_ws, s);
            SlotList sl = sorted_slots(sort_ws, a.batch, 31);
            order = sl.idx;
            order_count = sl.prefix + sl.bucket0;
        }
        cudaMemsetAsync(counters + CNT_L1_NEXT, 0, sizeof(int), s);
        KScope k(K_LU_L1, s);
        if (dm) {
            if (tall) lu_l1_kernel<true, true><<<grid, L1_NT, smem, s>>>(a, counters, bins, nb, rd, pt, order, order_count, df);
            else lu_l1_kernel<true, false><<<grid, L1_NT, smem, s>>>(a, counters, bins, nb, rd, pt, order, order_count, df);
        } else {
            if (tall) lu_l1_kernel<false, true><<<grid, L1_NT, smem, s>>>(a, counters, bins, nb, rd, pt, order, order_count, df);
            else lu_l1_kernel<false, false><<<grid, L1_NT, smem, s>>>(a, counters, bins, nb, rd, pt, order, order_count, df);
        }
    };
    if (tuning().l1_rows > L1_MAX_ROWS) one(BIN_L1T, true);
    one(BIN_L1, false);
}

// the grid-wide tier's list in LPT order (largest first, buckets of 32 in
// the cube-root key): every kernel of the tier walks slots in this order, so
// the dynamic queues hand out the biggest panels / strips first
// With two parts the sorted list is dealt alternately (part p gets the
// entries t = p, p + 2, ...: both halves LPT-ordered and flop-balanced); each
// part's count goes to its own counters block.
__global__ void set_bin_list_kernel(const int *__restrict__ sorted, const int *__restrict__ count_ptr,
                                    int *__restrict__ dst, int *__restrict__ dst_b, int *__restrict__ cnt_a,
                                    int *__restrict__ cnt_b) {
    const int count = *count_ptr;
    const int parts = dst_b ? 2 : 1;
    for (int t = blockIdx.x * blockDim.x + threadIdx.x; t < count; t += gridDim.x * blockDim.x) {
        if (parts == 1 || !(t & 1)) dst[t / parts] = sorted[t];
        else dst_b[t / 2] = sorted[t];
    }
    if (parts == 2 && blockIdx.x == 0 && threadIdx.x == 0) {
        *cnt_a = (count + 1) / 2;
        *cnt_b = count / 2;
    }
}

void launch_lu_large(const GetrfArgs &a, int *counters, const int *bins_c, int *tile_off, void *plans_v,
                     void *outer_plans_v, cudaStream_t s, int *keys, int *sort_ws, PartWork *pw) {
    int *bins = const_cast<int *>(bins_c);
    const Tuning &tu = tuning();
    // two parts (the LPT list dealt alternately) on two streams: one part's
    // latency-bound panels / strips / interchanges overlap the other part's
    // trailing GEMMs (two-level path only; see below)
    const bool two_parts = pw && pw->side && tu.parts == 2 && keys && sort_ws;
    if (keys && sort_ws) {
        cudaMemsetAsync(keys, 0, (size_t)a.batch * sizeof(int), s);
        const int g = (a.batch + 255) / 256;
        {
            KScope k(K_MISC, s);
            l1_key_kernel<<<g < 1024 ? g : 1024, 256, 0, s>>>(a, counters, bins, keys, BIN_L);
        }
        launch_size_sort(keys, a.batch, sort_ws, s);
        SlotList sl = sorted_slots(sort_ws, a.batch, 31);
        if (two_parts) cudaMemsetAsync(pw->counters, 0, CNT_INTS * sizeof(int), s);
        KScope k(K_MISC, s);
        set_bin_list_kernel<<<g < 1024 ? g : 1024, 256, 0, s>>>(
            sl.idx, sl.prefix + sl.bucket0, bins + (size_t)BIN_L * a.batch, two_parts ? pw->list : nullptr,
            counters + CNT_BIN0 + BIN_L, two_parts ? pw->counters + CNT_BIN0 + BIN_L : nullptr);
    }
    SwapPlan *plans = reinterpret_cast<SwapPlan *>(plans_v);
    const int nb = clamp_nb(tu.nb);
    const int Kmax = a.max_m < a.max_n ? a.max_m : a.max_n;
    // shared-memory panel rows: (rows|1) * nb doubles within the opt-in limit
    int smem_rows = tu.panel_rows;
    const int cap_rows = (int)((200 * 1024) / (sizeof(double) * nb)) - 1;
    if (smem_rows > cap_rows) smem_rows = cap_rows;
    if (smem_rows > a.max_m) smem_rows = a.max_m;
    size_t psmem = (size_t)((smem_rows | 1) + 1) * nb * sizeof(double);
    smem_optin(panel_kernel, psmem);
    const int sms = num_sms();
    int grid_p = sms * 2;
    if (grid_p > a.batch) grid_p = a.batch;
    smem_optin(panel_win_kernel<256>, sizeof(PanelWinSmem<8>));
    smem_optin(panel_win_kernel<512>, sizeof(PanelWinSmem<16>));
    smem_optin(panel_win_kernel<1024>, sizeof(PanelWinSmem<32>));
    int grid_w = sms * 2;
    if (grid_w > a.batch) grid_w = a.batch;
    const int chunks_per = (a.max_n + SW_COLS - 1) / SW_COLS;
    long long sw_items = (long long)a.batch * chunks_per;
    int grid_s = sms * 8;
    if (grid_s > sw_items) grid_s = (int)sw_items;
    const size_t sw_smem = (size_t)(nb * (nb + 1) + 2 * nb * (SW_COLS + 1)) * sizeof(double);
    smem_optin(swap_trsm_kernel, sw_smem);
    const int *listL = bins + (size_t)BIN_L * a.batch;
    const bool fused = tu.panel_win && tu.strip && a.max_m <= PW_MAX_ROWS;
    unsigned long long *ph = tu.phase_timing ? reinterpret_cast<unsigned long long *>(counters + CNT_PHASE0) : nullptr;
    const int st_chunks = (a.max_n + ST_COLS - 1) / ST_COLS;
    const size_t st_smem = strip_smem_bytes(nb);
    if (fused) {
        if (tu.dmma) smem_optin(strip_kernel<true>, st_smem);
        else smem_optin(strip_kernel<false>, st_smem);
    }
    // deferred left-block interchanges (strip path only): one pass at the end
    const int lsw_bufd = lsw_buf_doubles(a.max_m);
    const size_t lsw_smem = (size_t)lsw_bufd * sizeof(double) + 2 * (size_t)a.max_m * sizeof(int);
    const int nbo = (tu.nb_outer / nb) * nb;
    // two-level blocking (outer blocks of nbo columns) on the fused path; it
    // always defers the interchanges of the columns left of the outer block
    const bool outer = fused && nbo > nb && nbo <= NB_OUTER_MAX && lsw_smem <= 200 * 1024;
    const bool defer = fused && (tu.defer || outer) && lsw_smem <= 200 * 1024;
    if (defer) {
        smem_optin(left_swaps_kernel, lsw_smem);
    }
    if (outer) {
        OuterPlan *oplans = reinterpret_cast<OuterPlan *>(outer_plans_v);
        smem_optin(outer_swap_trsm_kernel<64>, OsCfg<64>::SMEM);
        smem_optin(outer_swap_trsm_kernel<32>, OsCfg<32>::SMEM);
        const bool os32 = tu.outer_cols == 32;
        smem_optin(xgemm_sched_kernel<OuterTrailProb, 0, 0, 8>, BIG_SMEM);
        smem_optin(xgemm_sched_kernel<OuterTrailProb, 0, 0, 16>, BIG_SMEM);
        smem_optin(xgemm_ws_kernel<OuterTrailProb, 0, 0>, BIG_SMEM);
        const int in_chunks = (nbo + ST_COLS - 1) / ST_COLS;
        // one part = one list of tier-L slots with its own counters block
        // (count, queues), plan slots, tile offsets and stream
        // few-large batches: the inner trailing update as a grid-wide GEMM
        // (tuning split_strip: 1 = always, 2 = auto when the batch has at most
        // SPLIT_BATCH matrices, 0 = never)
        const bool split = tu.split_strip == 1 || (tu.split_strip == 2 && a.batch <= SPLIT_BATCH);
        if (split) {
            gemm_smem_optin(gemm_sched_kernel<InnerTrailProb, true>);
            gemm_smem_optin(gemm_sched_kernel<InnerTrailProb, false>);
        }
        auto run_part = [&](int *cnt, int *bns, SwapPlan *pl, OuterPlan *opl, int *toff, cudaStream_t st, int gdiv) {
            const int *listP = bns + (size_t)BIN_L * a.batch;
            const int *cnt_ptr = cnt + CNT_BIN0 + BIN_L;
            const int gs = sms / gdiv > 0 ? sms / gdiv : 1;
            const int gw = grid_w / gdiv > 0 ? grid_w / gdiv : 1;
            for (int J = 0; J < Kmax; J += nbo) {
                for (int j = J; j < Kmax && j < J + nbo; j += nb) {
                    {
                        KScope k(K_PANEL, st);
                        launch_panel_win(a.max_m - j, gw, a, cnt, bns, j, nb, pl, cnt + CNT_STRIPQ, st);
                    }
                    {
                        KScope k(K_STRIP, st);
                        const int dg = split ? 0 : 1;
                        if (tu.dmma) strip_kernel<true><<<gs * 3, G_NT, st_smem, st>>>(
                            a, cnt, bns, pl, cnt + CNT_STRIPQ, j, nb, in_chunks, ph, 1, J, J + nbo, dg);
                        else strip_kernel<false><<<gs * 3, G_NT, st_smem, st>>>(
                            a, cnt, bns, pl, cnt + CNT_STRIPQ, j, nb, in_chunks, ph, 1, J, J + nbo, dg);
                    }
                    if (split) {
                        InnerTrailProb IP{a, listP, j, nb, J, J + nbo};
                        {
                            KScope k(K_GEMM_SCAN, st);
                            gemm_scan_kernel<InnerTrailProb><<<1, 1024, 0, st>>>(IP, -1, cnt_ptr, toff);
                        }
                        KScope k(K_STRIP, st);
                        if (tu.dmma)
                            gemm_sched_kernel<InnerTrailProb, true><<<gs * 3, G_NT, GEMM_SMEM, st>>>(IP, -1, cnt_ptr, toff);
                        else
                            gemm_sched_kernel<InnerTrailProb, false><<<gs * 3, G_NT, GEMM_SMEM, st>>>(IP, -1, cnt_ptr, toff);
                    }
                }
                {
                    KScope k(K_MISC, st);
                    int g = (a.batch + OP_NT / 32 - 1) / (OP_NT / 32);
                    if (g > gs * 8) g = gs * 8;
                    outer_plan_kernel<<<g, OP_NT, 0, st>>>(a, cnt, bns, J, nbo, opl, cnt + CNT_OUTQ);
                }
                {
                    KScope k(K_GEMM_SCAN, st);
                    if (os32)
                        scan_units_kernel<OuterStrips<32>><<<1, 1024, 0, st>>>(
                            OuterStrips<32>{a, listP, J, nbo}, SlotList{nullptr, cnt_ptr, 0}, a.batch, toff);
                    else
                        scan_units_kernel<OuterStrips<64>><<<1, 1024, 0, st>>>(
                            OuterStrips<64>{a, listP, J, nbo}, SlotList{nullptr, cnt_ptr, 0}, a.batch, toff);
                }
                {
                    KScope k(K_OUTER_TRSM, st);
                    if (os32)
                        outer_swap_trsm_kernel<32><<<2 * gs, OS_NT, OsCfg<32>::SMEM, st>>>(a, cnt, bns, opl, toff, J, nbo);
                    else
                        outer_swap_trsm_kernel<64><<<gs, OS_NT, OsCfg<64>::SMEM, st>>>(a, cnt, bns, opl, toff, J, nbo);
                }
                OuterTrailProb P{a, listP, J, nbo};
                {
                    KScope k(K_GEMM_SCAN, st);
                    xgemm_scan_kernel<OuterTrailProb><<<1, 1024, 0, st>>>(P, -1, cnt_ptr, toff);
                }
                KScope k(K_GEMM_TRAIL, st);
                if (tu.xgemm_warps == 9)
                    xgemm_ws_kernel<OuterTrailProb, 0, 0><<<gs, XWS_NT, BIG_SMEM, st>>>(P, -1, cnt_ptr, toff,
                                                                                       tu.xgemm_tma);
                else if (tu.xgemm_warps == 16)
                    xgemm_sched_kernel<OuterTrailProb, 0, 0, 16><<<gs * XGEMM_MINB, 512, BIG_SMEM, st>>>(P, -1, cnt_ptr,
                                                                                                     toff);
                else
                    xgemm_sched_kernel<OuterTrailProb, 0, 0, 8><<<gs * XGEMM_MINB, 256, BIG_SMEM, st>>>(P, -1, cnt_ptr,
                                                                                                    toff);
            }
            if (Kmax > nbo) {  // deferred left-block interchanges of this part
                cudaMemsetAsync(cnt + CNT_LSWQ, 0, sizeof(int), st);
                KScope k(K_LEFT_SWAPS, st);
                int grid = 2 * gs;
                if (grid > a.batch) grid = a.batch;
                left_swaps_kernel<<<grid, LSW_NT, lsw_smem, st>>>(a, cnt, bns, nbo, a.max_m, lsw_bufd, cnt + CNT_LSWQ);
            }
        };
        if (two_parts) {
            const size_t half = ((size_t)a.batch + 1) / 2;
            cudaEventRecord(pw->fork, s);
            cudaStreamWaitEvent(pw->side, pw->fork, 0);
            const int gdiv = tu.part_grid == 2 ? 2 : 1;
            run_part(counters, bins, plans, oplans, tile_off, s, gdiv);
            run_part(pw->counters, pw->list - (size_t)BIN_L * a.batch, plans + half, oplans + half, pw->tile_off,
                     pw->side, gdiv);
            cudaEventRecord(pw->join, pw->side);
            cudaStreamWaitEvent(s, pw->join, 0);
        } else {
            run_part(counters, bins, plans, oplans, tile_off, s, 1);
        }
        return;
    } else
    for (int j = 0; j < Kmax; j += nb) {
        if (tu.panel_win) {
            KScope k(K_PANEL, s);
            launch_panel_win(a.max_m - j, grid_w, a, counters, bins, j, nb, plans, counters + CNT_STRIPQ, s);
        } else {
            KScope k(K_PANEL, s);
            panel_kernel<<<grid_p, P_NT, psmem, s>>>(a, counters, bins, j, nb, smem_rows);
        }
        if (fused) {
            KScope k(K_STRIP, s);
            if (tu.dmma) strip_kernel<true><<<sms * 3, G_NT, st_smem, s>>>(a, counters, bins, plans,
                                                                             counters + CNT_STRIPQ, j, nb, st_chunks, ph,
                                                                             defer, -1, 1 << 30);
            else strip_kernel<false><<<sms * 3, G_NT, st_smem, s>>>(a, counters, bins, plans,
                                                                      counters + CNT_STRIPQ, j, nb, st_chunks, ph,
                                                                      defer, -1, 1 << 30);
            continue;
        }
        cudaMemsetAsync(counters + CNT_PANELQ, 0, sizeof(int), s);  // no strip kernel resets it on this path
        {
            KScope k(K_SWAP_TRSM, s);
            swap_trsm_kernel<<<grid_s, SW_NT, sw_smem, s>>>(a, counters, bins, j, nb, chunks_per);
        }
        TrailingProb P{a, listL, j, nb};
        {
            KScope k(K_GEMM_SCAN, s);
            gemm_scan_kernel<TrailingProb><<<1, 1024, 0, s>>>(P, -1, counters + CNT_BIN0 + BIN_L, tile_off);
        }
        {
            KScope k(K_GEMM_TRAIL, s);
            if (tu.dmma) {
                gemm_smem_optin(gemm_sched_kernel<TrailingProb, true>);
                gemm_sched_kernel<TrailingProb, true><<<sms * 3, G_NT, GEMM_SMEM, s>>>(
                    P, -1, counters + CNT_BIN0 + BIN_L, tile_off);
            } else {
                gemm_smem_optin(gemm_sched_kernel<TrailingProb, false>);
                gemm_sched_kernel<TrailingProb, false><<<sms * 3, G_NT, GEMM_SMEM, s>>>(
                    P, -1, counters + CNT_BIN0 + BIN_L, tile_off);
            }
        }
    }
    const int lnb = outer ? nbo : nb;  // block width of the deferred left interchanges
    if (defer && Kmax > lnb) {
        cudaMemsetAsync(counters + CNT_LSWQ, 0, sizeof(int), s);
        KScope k(K_LEFT_SWAPS, s);
        int grid = sms * 2;
        if (grid > a.batch) grid = a.batch;
        left_swaps_kernel<<<grid, LSW_NT, lsw_smem, s>>>(a, counters, bins, lnb, a.max_m, lsw_bufd,
                                                        counters + CNT_LSWQ);
    }
}

}  // namespace irr

// laswp_vb.cu -- irrLASWP (§IV-F) as an exported building block.
//
// "We begin by rehearsing the row interchanges on auxiliary ... single-column
// matrices ... initialized as 0, 1, 2, ...": each CTA composes the
// interchanges k1..k2-1 on an index list in shared memory (no global
// workspace, so the call stays asynchronous), compresses it to the
// list of rows that actually move, and then moves every such row exactly once
// per column (gather into shared memory, scatter back).  The widths are per
// matrix (DCWI: columns [Aj, Aj + min(max_n, n_i - Aj))).
#include "irr_internal.cuh"
#include "sched.cuh"

namespace irr {

constexpr int LS_NT = 256;
constexpr int LS_COLS = 32;
constexpr int LS_SPAN_MAX = 4096;  // interchanges per launch (shared-memory plan: 44 B each)

struct LaswpArgs {
    int max_n;
    const int *n;
    double *const *A;
    int Ai, Aj;
    const int *lda;
    int k1, k2;
    const int *kcount;
    int *const *ipiv;
    int batch;
    const int *mask;
    int chunks;
};

struct LaswpUnits {
    LaswpArgs g;
    __device__ int units(int i) const {
        if (g.mask && g.mask[i] < 0) return 0;
        const int ncol = imin(g.max_n, g.n[i] - g.Aj);
        const int kend = imin(g.k2, g.kcount[i]);
        if (ncol <= 0 || kend <= g.k1) return 0;
        return (ncol + LS_COLS - 1) / LS_COLS;
    }
};

// WALK = false: DCWI grid over batch x chunks of the required width;
// WALK = true : only the (matrix, chunk) units that exist (device schedule).
template <bool WALK>
__global__ void __launch_bounds__(LS_NT) laswp_kernel(LaswpArgs g, SlotList sl, const int *units_off) {
    extern __shared__ __align__(16) unsigned char ls_smem[];
    const int span = g.k2 - g.k1;
    int *top_src = (int *)ls_smem;             // [span]
    int *bot_pos = top_src + span;             // [span]
    int *bot_src = bot_pos + span;             // [span]
    int *mv_dst = bot_src + span;              // [2 span]
    int *mv_src = mv_dst + 2 * span;           // [2 span]
    double *vals = (double *)(((uintptr_t)(mv_src + 2 * span) + 15) & ~(uintptr_t)15);  // [2 span]
    __shared__ int nbot_s, nmov_s;
    const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
    int last_i = -1;
    auto body = [&](int i, int q) {
        if (g.mask && g.mask[i] < 0) return;
        const int ncol = imin(g.max_n, g.n[i] - g.Aj);
        const int kend = imin(g.k2, g.kcount[i]);
        if (ncol <= 0 || kend <= g.k1) return;
        const int c0 = q * LS_COLS;
        if (c0 >= ncol) return;
        const int W = imin(LS_COLS, ncol - c0);
        const long lda = g.lda[i];
        double *A = g.A[i] + g.Ai + (size_t)g.Aj * lda;
        if (i != last_i) {
            __syncthreads();
            // ---- rehearsal on the index list (warp 0), positions relative to Ai
            if (warp == 0) {
                const int *ip = g.ipiv[i];
                const int nk = kend - g.k1;
                for (int t = lane; t < nk; t += 32) top_src[t] = g.k1 + t;
                int nbot = 0;
                __syncwarp();
                for (int t = 0; t < nk; ++t) {
                    const int k = g.k1 + t;
                    const int p = ip[k] - 1;
                    if (p == k) continue;
                    if (p >= g.k1 && p < kend) {
                        if (lane == 0) {
                            int x = top_src[t];
                            top_src[t] = top_src[p - g.k1];
                            top_src[p - g.k1] = x;
                        }
                    } else {
                        int found = -1;
                        for (int b0 = 0; b0 < nbot; b0 += 32) {
                            int b = b0 + lane;
                            unsigned mk = __ballot_sync(FULL, b < nbot && bot_pos[b] == p);
                            if (mk) { found = b0 + __ffs(mk) - 1; break; }
                        }
                        if (found < 0) {
                            found = nbot++;
                            if (lane == 0) { bot_pos[found] = p; bot_src[found] = p; }
                        }
                        if (lane == 0) {
                            int x = top_src[t];
                            top_src[t] = bot_src[found];
                            bot_src[found] = x;
                        }
                    }
                    __syncwarp();
                }
                // compress to the rows that move
                int nmov = 0;
                for (int b0 = 0; b0 < nk; b0 += 32) {
                    const int t = b0 + lane;
                    const bool mv = t < nk && top_src[t] != g.k1 + t;
                    unsigned mk = __ballot_sync(FULL, mv);
                    if (mv) {
                        int o = nmov + __popc(mk & ((1u << lane) - 1));
                        mv_dst[o] = g.k1 + t;
                        mv_src[o] = top_src[t];
                    }
                    nmov += __popc(mk);
                }
                for (int b0 = 0; b0 < nbot; b0 += 32) {
                    const int b = b0 + lane;
                    const bool mv = b < nbot && bot_src[b] != bot_pos[b];
                    unsigned mk = __ballot_sync(FULL, mv);
                    if (mv) {
                        int o = nmov + __popc(mk & ((1u << lane) - 1));
                        mv_dst[o] = bot_pos[b];
                        mv_src[o] = bot_src[b];
                    }
                    nmov += __popc(mk);
                }
                if (lane == 0) { nbot_s = nbot; nmov_s = nmov; }
            }
            last_i = i;
            __syncthreads();
        }
        const int nmov = nmov_s;
        for (int c = 0; c < W; ++c) {
            double *col = A + (size_t)(c0 + c) * lda;
            for (int e = tid; e < nmov; e += LS_NT) vals[e] = col[mv_src[e]];
            __syncthreads();
            for (int e = tid; e < nmov; e += LS_NT) col[mv_dst[e]] = vals[e];
            __syncthreads();
        }
    };
    if (WALK) {
        walk_units(sl, g.batch, units_off, body);
    } else {
        const long long total = (long long)g.batch * g.chunks;
        for (long long w = blockIdx.x; w < total; w += gridDim.x) {
            const int i = (int)(w / g.chunks), q = (int)(w - (long long)i * g.chunks);
            body(i, q);
        }
    }
}

size_t laswp_smem(int span) {
    return (size_t)span * 7 * sizeof(int) + 16 + (size_t)span * 2 * sizeof(double);
}

// units_off: optional int[batch+1] workspace -> device-scheduled walk over
// the slots of `sl`; nullptr -> DCWI grid (the exported irr_laswp has no workspace).
void launch_laswp_masked(int max_n, const int *n, double *const *A, int Ai, int Aj, const int *lda, int k1, int k2,
                         const int *kcount, int *const *ipiv, int batch, const int *mask, cudaStream_t s,
                         int *units_off, SlotList sl) {
    if (batch <= 0 || max_n <= 0 || k2 <= k1) return;
    // long pivot ranges (the few-large regime): applied in consecutive
    // pieces, which is the same sequence of interchanges (stream-ordered)
    if (k2 - k1 > LS_SPAN_MAX) {
        for (int a = k1; a < k2; a += LS_SPAN_MAX)
            launch_laswp_masked(max_n, n, A, Ai, Aj, lda, a, a + LS_SPAN_MAX < k2 ? a + LS_SPAN_MAX : k2, kcount,
                                ipiv, batch, mask, s, units_off, sl);
        return;
    }
    LaswpArgs g{max_n, n, A, Ai, Aj, lda, k1, k2, kcount, ipiv, batch, mask, (max_n + LS_COLS - 1) / LS_COLS};
    size_t smem = laswp_smem(k2 - k1);
    if (units_off) {
        smem_optin(laswp_kernel<true>, smem);
        {
            KScope k(K_GEMM_SCAN, s);
            scan_units_kernel<LaswpUnits><<<1, 1024, 0, s>>>(LaswpUnits{g}, sl, batch, units_off);
        }
        KScope k(K_LASWP, s);
        laswp_kernel<true><<<num_sms() * 4, LS_NT, smem, s>>>(g, sl, units_off);
        return;
    }
    smem_optin(laswp_kernel<false>, smem);
    long long total = (long long)batch * g.chunks;
    int grid = num_sms() * 4;
    if (total < grid) grid = (int)total;
    KScope k(K_LASWP, s);
    laswp_kernel<false><<<grid, LS_NT, smem, s>>>(g, all_slots(), nullptr);
}

void launch_laswp(int max_n, const int *n, double *const *A, int Ai, int Aj, const int *lda, int k1, int k2,
                  const int *kcount, int *const *ipiv, int batch, cudaStream_t s) {
    launch_laswp_masked(max_n, n, A, Ai, Aj, lda, k1, k2, kcount, ipiv, batch, nullptr, s, nullptr, all_slots());
}

}  // namespace irr

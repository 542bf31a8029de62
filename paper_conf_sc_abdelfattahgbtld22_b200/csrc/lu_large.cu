// lu_large.cu -- tier L: blocked right-looking LU with partial pivoting on
// the matrices too large for one shared-memory tile.
//
// One iteration per panel of nb columns (Fig. 1), written for the
// largest matrix (DCWI: the host loops over ITERATIONS of the largest
// matrix, never over matrices; each kernel infers full / partial / no work):
//   a4.1 panel_kernel     fused irrGETF2 on the (m_i - j) x ib panel, staged in
//                         shared memory when it fits, else in place
//   a4.2+a4.3 swap_trsm   the panel's row interchanges, "rehearsed" on an
//                         index list first and then applied once per
//                         moved row to the left and right column blocks; the
//                         right block is solved in the same pass:
//                         U12 <- L11^-1 P A12 (irrLASWP + irrTRSM fused)
//   a4.4 gemm            A22 -= L21 U12 through the device tile schedule
#include "gemm_core.cuh"
#include "panel.cuh"

namespace irr {

constexpr int P_NT = 512;
constexpr int NBMAX = 64;     // largest supported panel width
constexpr int SW_COLS = 32;   // columns per swap/TRSM work item
constexpr int SW_NT = 128;

// ------------------------------------------------------------------ a4.1 panel
__global__ void __launch_bounds__(P_NT) panel_kernel(GetrfArgs a, const int *__restrict__ counters,
                                                     const int *__restrict__ bins, int j, int nb, int smem_rows) {
    extern __shared__ __align__(16) double sp[];
    __shared__ PanelScratch sc;
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
            P = sp;
            for (int c = warp; c < ib; c += NW)
                for (int r = lane; r < rows; r += 32) P[r + c * ldp] = gP[r + (size_t)c * ld];
            __syncthreads();
        } else {
            P = gP;
            ldp = ld;
        }
        int z = panel_getf2<P_NT>(P, ldp, 0, rows, 0, ib, 0, ib, piv_s, sc);
        if (staged) {
            for (int c = warp; c < ib; c += NW)
                for (int r = lane; r < rows; r += 32) gP[r + (size_t)c * ld] = P[r + c * ldp];
        }
        if (tid < ib) a.ipiv[i][j + tid] = j + piv_s[tid] + 1;
        if (tid == 0 && z && a.info[i] == 0) a.info[i] = j + z;
        __syncthreads();
    }
}

// ------------------------------------------------------------------ a4.2 + a4.3
// Work item = (tier-L slot, column chunk of SW_COLS).  Chunks 0..nleft-1 cover
// the columns left of the panel [0, j) (interchanges only), the rest cover
// [j+ib, n) (interchanges + forward substitution with the unit L11).
__global__ void __launch_bounds__(SW_NT) swap_trsm_kernel(GetrfArgs a, const int *__restrict__ counters,
                                                          const int *__restrict__ bins, int j, int nb,
                                                          int chunks_per) {
    extern __shared__ __align__(16) double sw_smem[];
    // L11: nb x (nb+1); top: rows j..j+ib-1 of the chunk; bot: moved rows below
    double *L11s = sw_smem;
    double *tops = L11s + nb * (nb + 1);
    double *bots = tops + nb * (SW_COLS + 1);
#define L11(r, c) L11s[(r) * (nb + 1) + (c)]
#define top(t, c) tops[(t) * (SW_COLS + 1) + (c)]
#define bot(b, c) bots[(b) * (SW_COLS + 1) + (c)]
    __shared__ int top_src[NBMAX];                // source row of position j+t
    __shared__ int bot_pos[NBMAX], bot_src[NBMAX];
    __shared__ int nbot_s;
    const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
    const int count = counters[CNT_BIN0 + BIN_L];
    const int *list = bins + (size_t)BIN_L * a.batch;
    const long long total = (long long)count * chunks_per;
    int last_i = -1;
    for (long long w = blockIdx.x; w < total; w += gridDim.x) {
        const int slot = (int)(w / chunks_per), q = (int)(w - (long long)slot * chunks_per);
        const int i = list[slot];
        const int mi = a.m[i], ni = a.n[i], ld = a.ld[i];
        const int K = mi < ni ? mi : ni;
        if (j >= K) continue;
        const int ib = K - j < nb ? K - j : nb;
        const int c1 = j + ib;
        const int nleft = (j + SW_COLS - 1) / SW_COLS;
        const int nright = (ni - c1 + SW_COLS - 1) / SW_COLS;
        if (q >= nleft + nright) continue;
        const bool right = q >= nleft;
        const int cbeg = right ? c1 + (q - nleft) * SW_COLS : q * SW_COLS;
        const int cend = right ? imin(ni, cbeg + SW_COLS) : imin(j, cbeg + SW_COLS);
        const int W = cend - cbeg;
        double *gA = a.A[i];
        const int *ip = a.ipiv[i];
        // ---- rehearsal: compose the ib interchanges on an index list (warp 0)
        if (i != last_i) {
            __syncthreads();
            if (warp == 0) {
                for (int t = lane; t < ib; t += 32) top_src[t] = j + t;
                int nbot = 0;
                __syncwarp();
                for (int t = 0; t < ib; ++t) {
                    const int p = ip[j + t] - 1;  // absolute row
                    if (p == j + t) continue;
                    if (p < c1) {
                        if (lane == 0) {
                            int x = top_src[t];
                            top_src[t] = top_src[p - j];
                            top_src[p - j] = x;
                        }
                    } else {
                        // find p in the bottom list (warp-parallel search)
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
                if (lane == 0) nbot_s = nbot;
            }
            if (right) {
                for (int e = tid; e < ib * ib; e += SW_NT) {
                    int r = e % ib, c = e / ib;
                    L11(r, c) = gA[j + r + (size_t)(j + c) * ld];
                }
            }
            last_i = right ? i : -1;  // L11 only valid when loaded
            __syncthreads();
        }
        const int nbot = nbot_s;
        // ---- gather the moved rows of this chunk (reads before any write)
        for (int e = tid; e < ib * W; e += SW_NT) {
            int t = e % ib, c = e / ib;
            top(t, c) = gA[top_src[t] + (size_t)(cbeg + c) * ld];
        }
        for (int e = tid; e < nbot * W; e += SW_NT) {
            int b = e % nbot, c = e / nbot;
            bot(b, c) = gA[bot_src[b] + (size_t)(cbeg + c) * ld];
        }
        __syncthreads();
        // ---- forward substitution on the top block (right chunks), one thread per column
        if (right && tid < W) {
            for (int s = 0; s < ib; ++s) {
                const double x = top(s, tid);
                for (int r = s + 1; r < ib; ++r) top(r, tid) = fma(-L11(r, s), x, top(r, tid));
            }
        }
        __syncthreads();
        // ---- write back
        for (int e = tid; e < ib * W; e += SW_NT) {
            int t = e % ib, c = e / ib;
            gA[j + t + (size_t)(cbeg + c) * ld] = top(t, c);
        }
        for (int e = tid; e < nbot * W; e += SW_NT) {
            int b = e % nbot, c = e / nbot;
            gA[bot_pos[b] + (size_t)(cbeg + c) * ld] = bot(b, c);
        }
        __syncthreads();
    }
#undef L11
#undef top
#undef bot
}

// ------------------------------------------------------------------ a4.4 problem
struct TrailingProb {
    GetrfArgs a;
    const int *list;
    int j, nb;
    __device__ bool get(int slot, GemmDesc &d) const {
        const int i = list[slot];
        const int mi = a.m[i], ni = a.n[i];
        const int K = mi < ni ? mi : ni;
        d.m = 0; d.n = 0; d.k = 0;
        if (j >= K) return false;
        const int ib = K - j < nb ? K - j : nb;
        const int c1 = j + ib;
        if (c1 >= mi || c1 >= ni) return false;
        const long ld = a.ld[i];
        double *A = a.A[i];
        d.A = A + c1 + (size_t)j * ld; d.lda = ld; d.ta = 0;
        d.B = A + j + (size_t)c1 * ld; d.ldb = ld; d.tb = 0;
        d.C = A + c1 + (size_t)c1 * ld; d.ldc = ld;
        d.m = mi - c1; d.n = ni - c1; d.k = ib;
        d.alpha = -1.0; d.beta = 1.0;
        return true;
    }
};

void launch_lu_large(const GetrfArgs &a, int *counters, const int *bins, int *tile_off, cudaStream_t s) {
    const Tuning &tu = tuning();
    int nb = tu.nb;
    if (nb < 1) nb = 1;
    if (nb > NBMAX) nb = NBMAX;
    const int Kmax = a.max_m < a.max_n ? a.max_m : a.max_n;
    // shared-memory panel rows: (rows|1) * nb doubles within the opt-in limit
    int smem_rows = tu.panel_rows;
    const int cap_rows = (int)((200 * 1024) / (sizeof(double) * nb)) - 1;
    if (smem_rows > cap_rows) smem_rows = cap_rows;
    int rows_need = a.max_m;
    if (smem_rows > rows_need) smem_rows = rows_need;
    size_t psmem = (size_t)((smem_rows | 1) + 1) * nb * sizeof(double);
    static size_t attr_max = 0;
    if (psmem > attr_max) {
        cudaFuncSetAttribute(panel_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)psmem);
        attr_max = psmem;
    }
    const int sms = num_sms();
    int grid_p = sms * 2;
    if (grid_p > a.batch) grid_p = a.batch;
    const int chunks_per = (a.max_n + SW_COLS - 1) / SW_COLS + 1;
    long long sw_items = (long long)a.batch * chunks_per;
    int grid_s = sms * 8;
    if (grid_s > sw_items) grid_s = (int)sw_items;
    const size_t sw_smem = (size_t)(nb * (nb + 1) + 2 * nb * (SW_COLS + 1)) * sizeof(double);
    static size_t sw_attr = 0;
    if (sw_smem > 48 * 1024 && sw_smem > sw_attr) {
        cudaFuncSetAttribute(swap_trsm_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)sw_smem);
        sw_attr = sw_smem;
    }
    const int *listL = bins + (size_t)BIN_L * a.batch;
    for (int j = 0; j < Kmax; j += nb) {
        {
            KScope k(K_PANEL, s);
            panel_kernel<<<grid_p, P_NT, psmem, s>>>(a, counters, bins, j, nb, smem_rows);
        }
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
            gemm_sched_kernel<TrailingProb><<<sms * 2, G_NT, 0, s>>>(P, -1, counters + CNT_BIN0 + BIN_L, tile_off);
        }
    }
}

}  // namespace irr

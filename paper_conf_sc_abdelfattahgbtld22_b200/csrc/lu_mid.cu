// lu_mid.cu -- tier M: one CTA per matrix, the whole matrix resident in shared
// memory.
//
// The fused irrGETF2 panel is only worthwhile while the data fits in
// shared memory ("the advantage ... is saving memory traffic"; the
// 192 KB of the A100 vs 64 KB of the MI100 decided the switch).  On
// B200 (227 KB per CTA) the whole matrix fits for m*n <= 24,576, so the full
// blocked right-looking LU (Fig. 1) runs on chip: A is read once and
// written once.  Per panel of NBM columns: fused panel (panel.cuh), in-place
// TRSM of the U12 row block, register-tiled GEMM update of the trailing
// matrix, all in shared memory.
#include "panel.cuh"
#include "gemm_core.cuh"  // dmma_8x8x4

namespace irr {

constexpr int NBM = 16;

// A22 -= L21 U12 in shared memory on the FP64 tensor core (tuning mid_dmma):
// warp tiles of 32 x 32 = 4 x 4 mma.sync.m8n8k4 tiles, the C fragments read
// from and written back to the resident matrix, K = ib <= NBM in steps of 4
// (A = -L21 so that D = C + A B).  Fragment layout of m8n8k4.f64 row.col:
// lane (g = lane / 4, t = lane % 4) holds A[g][t], B[t][g], C[g][2t, 2t + 1].
template <int NW>
__device__ __forceinline__ void mid_update_dmma(double *s, int lds, int j, int ib, int c1, int mi, int ni) {
    const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5, g = lane >> 2, t = lane & 3;
    const int Mr = mi - c1, Nc = ni - c1;
    const int tm = (Mr + 31) >> 5, tn = (Nc + 31) >> 5;
    for (int item = warp; item < tm * tn; item += NW) {
        const int rb = c1 + (item % tm) * 32, cb = c1 + (item / tm) * 32;
        double acc[4][4][2];
#pragma unroll
        for (int a4 = 0; a4 < 4; ++a4) {
            const int r = rb + 8 * a4 + g;
#pragma unroll
            for (int b4 = 0; b4 < 4; ++b4) {
                const int c = cb + 8 * b4 + 2 * t;
                acc[a4][b4][0] = (r < mi && c < ni) ? s[r + c * lds] : 0.0;
                acc[a4][b4][1] = (r < mi && c + 1 < ni) ? s[r + (c + 1) * lds] : 0.0;
            }
        }
        for (int kk = 0; kk < ib; kk += 4) {
            const bool kv = kk + t < ib;
            const int k = j + kk + t;
            double a[4], b[4];
#pragma unroll
            for (int a4 = 0; a4 < 4; ++a4) {
                const int r = rb + 8 * a4 + g;
                a[a4] = (kv && r < mi) ? -s[r + k * lds] : 0.0;
            }
#pragma unroll
            for (int b4 = 0; b4 < 4; ++b4) {
                const int c = cb + 8 * b4 + g;
                b[b4] = (kv && c < ni) ? s[k + c * lds] : 0.0;
            }
#pragma unroll
            for (int a4 = 0; a4 < 4; ++a4)
#pragma unroll
                for (int b4 = 0; b4 < 4; ++b4) dmma_8x8x4(acc[a4][b4][0], acc[a4][b4][1], a[a4], b[b4]);
        }
#pragma unroll
        for (int a4 = 0; a4 < 4; ++a4) {
            const int r = rb + 8 * a4 + g;
            if (r >= mi) continue;
#pragma unroll
            for (int b4 = 0; b4 < 4; ++b4) {
                const int c = cb + 8 * b4 + 2 * t;
                if (c < ni) s[r + c * lds] = acc[a4][b4][0];
                if (c + 1 < ni) s[r + (c + 1) * lds] = acc[a4][b4][1];
            }
        }
    }
}

// M_NT threads, MINB CTAs per SM (registers capped so the footprint-limited
// occupancy is reachable: M1 48 KB -> 4 CTAs, M2 96 KB -> 2, M3 192 KB -> 1)
template <int M_NT, int MINB>
__global__ void __launch_bounds__(M_NT, MINB) lu_mid_kernel(GetrfArgs a, const int *__restrict__ counters,
                                                      const int *__restrict__ bins, int bin,
                                                      unsigned long long *ph, int dmma) {
    extern __shared__ __align__(16) double s[];
    long long t0 = 0;
#define MID_PHASE(k)                                                                    \
    if (ph && threadIdx.x == 0) {                                                       \
        long long t1 = clock64();                                                       \
        atomicAdd(ph + (k), (unsigned long long)(t1 - t0));                             \
        t0 = t1;                                                                        \
    }
    __shared__ PanelScratch sc;
    __shared__ __align__(16) PanelRegScratch<M_NT / 32, NBM> prs;
    __shared__ int piv_s[NBM];
    const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
    constexpr int NW = M_NT / 32;
    const int count = counters[CNT_BIN0 + bin];
    const int *list = bins + (size_t)bin * a.batch;
    for (int t = blockIdx.x; t < count; t += gridDim.x) {
        const int i = list[t];
        const int mi = a.m[i], ni = a.n[i], ld = a.ld[i];
        double *__restrict__ gA = a.A[i];
        const int lds = mid_lds(mi);
        if (ph && tid == 0) t0 = clock64();
        // ---- load: the whole matrix in flight at once (cp.async)
        stage_block_async(s, lds, gA, ld, mi, ni, tid, M_NT);
        cp_async_commit();
        cp_async_wait<0>();
        __syncthreads();
        MID_PHASE(3)
        const int K = mi < ni ? mi : ni;
        int info = 0;
        int *gipiv = a.ipiv[i];
        for (int j = 0; j < K; j += NBM) {
            const int ib = K - j < NBM ? K - j : NBM;
            // ---- fused panel, interchanges applied to the full rows
            int z;
            if (mi - j <= 2 * M_NT) {
                // register-resident panel (1 barrier per column), then the
                // panel's interchanges on the other columns, one thread per column
                z = panel_regs<M_NT, 2, NBM>(s + j + j * lds, lds, mi - j, ib, piv_s, prs);
                for (int cc = tid; cc < ni; cc += M_NT) {
                    if (cc >= j && cc < j + ib) continue;
                    double *col = s + cc * lds;
                    for (int c = 0; c < ib; ++c) {
                        const int p = j + piv_s[c];
                        if (p != j + c) {
                            const double x = col[j + c];
                            col[j + c] = col[p];
                            col[p] = x;
                        }
                    }
                }
                __syncthreads();
                if (tid < ib) piv_s[tid] += j;
            } else {
                z = panel_getf2<M_NT>(s, lds, j, mi, j, ib, 0, ni, piv_s, sc);
            }
            if (z && !info) info = j + z;
            if (tid < ib) gipiv[j + tid] = piv_s[tid] + 1;
            MID_PHASE(4)
            const int c1 = j + ib;
            if (c1 >= ni) continue;
            // ---- U12 <- L11^-1 A12 (unit lower, in place), one thread per column
            for (int cc = c1 + tid; cc < ni; cc += M_NT) {
                double x[NBM];
#pragma unroll
                for (int q = 0; q < NBM; ++q) x[q] = (q < ib) ? s[j + q + cc * lds] : 0.0;
#pragma unroll
                for (int q = 0; q < NBM; ++q) {
#pragma unroll
                    for (int r = q + 1; r < NBM; ++r)
                        if (r < ib) x[r] = fma(-s[j + r + (j + q) * lds], x[q], x[r]);
                }
#pragma unroll
                for (int q = 0; q < NBM; ++q)
                    if (q < ib) s[j + q + cc * lds] = x[q];
            }
            __syncthreads();
            MID_PHASE(5)
            // ---- A22 -= L21 * U12 : DMMA warp tiles (mid_dmma), or warp tiles
            //      of 64 rows x 4 columns with the lane owning rows (lane, lane + 32)
            const int Mr = mi - c1, Nc = ni - c1;
            if (Mr > 0 && dmma) {
                mid_update_dmma<NW>(s, lds, j, ib, c1, mi, ni);
            } else if (Mr > 0) {
                const int nrt = (Mr + 63) >> 6, nct = (Nc + 3) >> 2;
                for (int item = warp; item < nrt * nct; item += NW) {
                    const int tr = item % nrt, tc = item / nrt;
                    const int r0 = c1 + tr * 64 + lane, cb = c1 + tc * 4;
                    const bool v0 = r0 < mi, v1 = r0 + 32 < mi;
                    double acc[2][4] = {{0, 0, 0, 0}, {0, 0, 0, 0}};
                    for (int kk = 0; kk < ib; ++kk) {
                        const double *Lc = s + (j + kk) * lds;
                        double a0 = v0 ? Lc[r0] : 0.0, a1 = v1 ? Lc[r0 + 32] : 0.0;
#pragma unroll
                        for (int p = 0; p < 4; ++p) {
                            double b = (cb + p < ni) ? s[j + kk + (cb + p) * lds] : 0.0;
                            acc[0][p] = fma(a0, b, acc[0][p]);
                            acc[1][p] = fma(a1, b, acc[1][p]);
                        }
                    }
#pragma unroll
                    for (int p = 0; p < 4; ++p) {
                        if (cb + p < ni) {
                            if (v0) s[r0 + (cb + p) * lds] -= acc[0][p];
                            if (v1) s[r0 + 32 + (cb + p) * lds] -= acc[1][p];
                        }
                    }
                }
            }
            __syncthreads();
            MID_PHASE(6)
        }
        // ---- store
        for (int c = warp; c < ni; c += NW)
            for (int r = lane; r < mi; r += 32) gA[r + (size_t)c * ld] = s[r + c * lds];
        if (tid == 0) a.info[i] = info;
        __syncthreads();
        MID_PHASE(7)
    }
#undef MID_PHASE
}

void launch_lu_mid(const GetrfArgs &a, const int *counters, const int *bins, int bin, int max_elems,
                   cudaStream_t s) {
    size_t smem = (size_t)max_elems * sizeof(double);
    int per_sm = (int)(220 * 1024 / (smem + 2048));
    if (per_sm < 1) per_sm = 1;
    if (per_sm > 4) per_sm = 4;
    int grid = num_sms() * per_sm;
    if (grid > a.batch) grid = a.batch;
    if (grid < 1) grid = 1;
    const int dm = tuning().mid_dmma;
    KScope k(K_LU_MID, s);
    unsigned long long *ph =
        tuning().phase_timing ? reinterpret_cast<unsigned long long *>(const_cast<int *>(counters) + CNT_PHASE0)
                              : nullptr;
    if (per_sm >= 4) {
        smem_optin(lu_mid_kernel<128, 4>, smem);
        lu_mid_kernel<128, 4><<<grid, 128, smem, s>>>(a, counters, bins, bin, ph, dm);
    } else if (per_sm >= 2) {
        smem_optin(lu_mid_kernel<256, 2>, smem);
        lu_mid_kernel<256, 2><<<grid, 256, smem, s>>>(a, counters, bins, bin, ph, dm);
    } else {
        smem_optin(lu_mid_kernel<256, 1>, smem);
        lu_mid_kernel<256, 1><<<grid, 256, smem, s>>>(a, counters, bins, bin, ph, dm);
    }
}

}  // namespace irr

// irr_getrs with one right-hand side per system (max_nrhs == 1): x <- U^-1
// L^-1 P^T b (PAPER.md L96 / L215, the GETRS composition).
//
// With one column the solve is a chain of n dependent steps streaming the
// n x n L\U once (8 n^2 bytes, AI 0.25 flop/B): HBM / latency bound, not a
// GEMM.  The strip kernel (getrs_strip.cu) spends one CTA per (system,
// 64-column strip) and its DMMA tiles on a single column; here one CTA of
// GV_THREADS owns one system:
//   * b and ipiv staged in shared memory, the interchanges applied in order by
//     one thread (smem only);
//   * substitution in 32-column blocks: warp 0 solves the 32 x 32 diagonal
//     triangle (staged in shared memory one block ahead) with x in registers
//     (lane i = row i of the block, shuffles broadcast the solved entry),
//     then every thread updates its rows below
//     (L) / above (U) with the block's 32 columns -- for a fixed column,
//     consecutive threads read consecutive rows (coalesced, each element of
//     L\U read exactly once).  Two barriers per 32 columns.
// U's diagonal is divided by (IEEE division, as the oracle), not inverted.
#include "irr_internal.cuh"

namespace irr {

constexpr int GV_THREADS = 128;
#ifndef GV_UNROLL
#define GV_UNROLL 8  // loads in flight per thread in the column updates
#endif
constexpr int kGvUnroll = GV_UNROLL;
#ifndef GV_MINB
#define GV_MINB 8  // 64 registers: 8 CTAs (32 warps) per SM
#endif

__global__ void __launch_bounds__(GV_THREADS, GV_MINB)
    getrs_vec_kernel(const int *__restrict__ n_, const int *__restrict__ nrhs_, const double *const *__restrict__ A,
                     const int *__restrict__ lda_, int *const *__restrict__ ipiv_, double *const *__restrict__ B,
                     const int *__restrict__ ldb_, const int *__restrict__ mask) {
    extern __shared__ double x[];  // n entries, then n ints of ipiv
    const int s = blockIdx.x;
    const int n = n_[s];
    if (mask[s] != 0 || n <= 0 || nrhs_[s] <= 0) return;
    const double *__restrict__ LU = A[s];
    const size_t lda = (size_t)lda_[s];
    double *__restrict__ b = B[s];
    const int *__restrict__ ip = ipiv_[s];
    int *sp = reinterpret_cast<int *>(x + n);
    const int t = threadIdx.x, lane = t & 31, warp = t >> 5;
    for (int i = t; i < n; i += GV_THREADS) {
        x[i] = b[i];
        sp[i] = __ldg(ip + i);
    }
    __syncthreads();
    if (t == 0)
        for (int k = 0; k < n; ++k) {
            const int p = sp[k] - 1;
            if (p != k) {
                const double v = x[k];
                x[k] = x[p];
                x[p] = v;
            }
        }
    __syncthreads();
    // forward: L unit lower.  The 32 x 32 diagonal tile of the next block is
    // staged in shared memory by all threads together with the current
    // block's trailing update (both only read L\U), so warp 0's dependent
    // chain reads it from shared memory and the registers stay low.
    __shared__ double tri[32 * 33];
    auto stage = [&](int jb, int w, bool lower) {
        for (int e = t; e < 32 * 32; e += GV_THREADS) {
            const int r = e & 31, k = e >> 5;
            const bool in = r < w && k < w && (lower ? k < r : k >= r);
            tri[r * 33 + k] = in ? LU[(size_t)(jb + r) + (size_t)(jb + k) * lda] : 0.0;
        }
    };
    stage(0, min(32, n), true);
    __syncthreads();
    for (int jb = 0; jb < n; jb += 32) {
        const int w = min(32, n - jb);
        if (warp == 0) {
            double xi = lane < w ? x[jb + lane] : 0.0;
#pragma unroll
            for (int k = 0; k < 31; ++k) {
                const double xk = __shfl_sync(0xffffffffu, xi, k);
                xi -= tri[lane * 33 + k] * xk;  // 0 unless k < lane < w
            }
            if (lane < w) x[jb + lane] = xi;
        }
        __syncthreads();
        for (int i = jb + w + t; i < n; i += GV_THREADS) {
            double acc = x[i];
            const double *col = LU + (size_t)i + (size_t)jb * lda;
#pragma unroll kGvUnroll
            for (int k = 0; k < w; ++k) acc -= col[(size_t)k * lda] * x[jb + k];
            x[i] = acc;
        }
        if (jb + 32 < n) stage(jb + 32, min(32, n - jb - 32), true);
        __syncthreads();
    }
    // backward: U upper, non-unit; blocks from the bottom
    const int nblk = (n + 31) / 32;
    stage((nblk - 1) * 32, n - (nblk - 1) * 32, false);
    __syncthreads();
    for (int q = nblk - 1; q >= 0; --q) {
        const int jb = q * 32, w = min(32, n - jb);
        if (warp == 0) {
            double xi = lane < w ? x[jb + lane] : 0.0;
#pragma unroll
            for (int k = 31; k >= 0; --k) {
                if (k < w) {
                    if (lane == k) xi = xi / tri[k * 33 + k];
                    const double xk = __shfl_sync(0xffffffffu, xi, k);
                    if (lane < k) xi -= tri[lane * 33 + k] * xk;
                }
            }
            if (lane < w) x[jb + lane] = xi;
        }
        __syncthreads();
        for (int i = t; i < jb; i += GV_THREADS) {
            double acc = x[i];
            const double *col = LU + (size_t)i + (size_t)jb * lda;
#pragma unroll kGvUnroll
            for (int k = 0; k < w; ++k) acc -= col[(size_t)k * lda] * x[jb + k];
            x[i] = acc;
        }
        if (q > 0) stage(jb - 32, 32, false);
        __syncthreads();
    }
    for (int i = t; i < n; i += GV_THREADS) b[i] = x[i];
}

bool getrs_vec_ok(int max_n) { return max_n > 0 && (size_t)max_n * 12 <= 200 * 1024; }

void launch_getrs_vec(int batch, int max_n, const int *n, const int *nrhs, const double *const *A, const int *lda,
                      int *const *ipiv, double *const *B, const int *ldb, const int *mask, cudaStream_t s) {
    const size_t smem = (size_t)max_n * 12;
    if (smem > 48 * 1024)
        cudaFuncSetAttribute(getrs_vec_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
    KScope k(K_GETRS, s);
    getrs_vec_kernel<<<batch, GV_THREADS, smem, s>>>(n, nrhs, A, lda, ipiv, B, ldb, mask);
}

}  // namespace irr

// irr_getrs with few right-hand sides per system (max_nrhs <= GV_MAX_NRHS;
// R = 1, 2 or 4 columns held per CTA): x <- U^-1 L^-1 P^T b (PAPER.md L96 / L215, the GETRS composition).
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
#ifndef GV_MAX_NRHS
#define GV_MAX_NRHS 4  // widest RHS block per CTA (R = 1, 2, 4); R = 8 measured slower than the strip path
#endif
#ifndef GV_UNROLL
#define GV_UNROLL 8  // loads in flight per thread in the column updates
#endif
constexpr int kGvUnroll = GV_UNROLL;
#ifndef GV_MINB
#define GV_MINB 8  // 64 registers: 8 CTAs (32 warps) per SM
#endif

template <int R>
__global__ void __launch_bounds__(GV_THREADS, GV_MINB)
    getrs_vec_kernel(const int *__restrict__ n_, const int *__restrict__ nrhs_, const double *const *__restrict__ A,
                     const int *__restrict__ lda_, int *const *__restrict__ ipiv_, double *const *__restrict__ B,
                     const int *__restrict__ ldb_, const int *__restrict__ mask) {
    extern __shared__ double x[];  // n x R (row i at x[i R]), then n ints of ipiv
    const int s = blockIdx.x;
    const int n = n_[s], nr = nrhs_[s];
    if (mask[s] != 0 || n <= 0 || nr <= 0) return;
    const double *__restrict__ LU = A[s];
    const size_t lda = (size_t)lda_[s];
    double *__restrict__ b = B[s];
    const size_t ldb = (size_t)ldb_[s];
    const int *__restrict__ ip = ipiv_[s];
    int *sp = reinterpret_cast<int *>(x + (size_t)n * R);
    const int t = threadIdx.x, lane = t & 31, warp = t >> 5;
    for (int i = t; i < n; i += GV_THREADS) {
#pragma unroll
        for (int r = 0; r < R; ++r) x[i * R + r] = r < nr ? b[(size_t)i + r * ldb] : 0.0;
        sp[i] = __ldg(ip + i);
    }
    __syncthreads();
    if (t == 0)
        for (int k = 0; k < n; ++k) {
            const int p = sp[k] - 1;
            if (p != k)
#pragma unroll
                for (int r = 0; r < R; ++r) {
                    const double v = x[k * R + r];
                    x[k * R + r] = x[p * R + r];
                    x[p * R + r] = v;
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
            double xi[R];
#pragma unroll
            for (int r = 0; r < R; ++r) xi[r] = lane < w ? x[(jb + lane) * R + r] : 0.0;
#pragma unroll
            for (int k = 0; k < 31; ++k) {
                const double l = tri[lane * 33 + k];  // 0 unless k < lane < w
#pragma unroll
                for (int r = 0; r < R; ++r) xi[r] -= l * __shfl_sync(0xffffffffu, xi[r], k);
            }
            if (lane < w)
#pragma unroll
                for (int r = 0; r < R; ++r) x[(jb + lane) * R + r] = xi[r];
        }
        __syncthreads();
        for (int i = jb + w + t; i < n; i += GV_THREADS) {
            double acc[R];
#pragma unroll
            for (int r = 0; r < R; ++r) acc[r] = x[i * R + r];
            const double *col = LU + (size_t)i + (size_t)jb * lda;
#pragma unroll kGvUnroll
            for (int k = 0; k < w; ++k) {
                const double l = col[(size_t)k * lda];
#pragma unroll
                for (int r = 0; r < R; ++r) acc[r] -= l * x[(jb + k) * R + r];
            }
#pragma unroll
            for (int r = 0; r < R; ++r) x[i * R + r] = acc[r];
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
            double xi[R];
#pragma unroll
            for (int r = 0; r < R; ++r) xi[r] = lane < w ? x[(jb + lane) * R + r] : 0.0;
#pragma unroll
            for (int k = 31; k >= 0; --k) {
                if (k < w) {
                    const double d = tri[k * 33 + k], u = tri[lane * 33 + k];
#pragma unroll
                    for (int r = 0; r < R; ++r) {
                        if (lane == k) xi[r] = xi[r] / d;
                        const double xk = __shfl_sync(0xffffffffu, xi[r], k);
                        if (lane < k) xi[r] -= u * xk;
                    }
                }
            }
            if (lane < w)
#pragma unroll
                for (int r = 0; r < R; ++r) x[(jb + lane) * R + r] = xi[r];
        }
        __syncthreads();
        for (int i = t; i < jb; i += GV_THREADS) {
            double acc[R];
#pragma unroll
            for (int r = 0; r < R; ++r) acc[r] = x[i * R + r];
            const double *col = LU + (size_t)i + (size_t)jb * lda;
#pragma unroll kGvUnroll
            for (int k = 0; k < w; ++k) {
                const double l = col[(size_t)k * lda];
#pragma unroll
                for (int r = 0; r < R; ++r) acc[r] -= l * x[(jb + k) * R + r];
            }
#pragma unroll
            for (int r = 0; r < R; ++r) x[i * R + r] = acc[r];
        }
        if (q > 0) stage(jb - 32, 32, false);
        __syncthreads();
    }
    for (int i = t; i < n; i += GV_THREADS)
#pragma unroll
        for (int r = 0; r < R; ++r)
            if (r < nr) b[(size_t)i + r * ldb] = x[i * R + r];
}

static int vec_r(int max_nrhs) { return max_nrhs <= 1 ? 1 : max_nrhs <= 2 ? 2 : max_nrhs <= 4 ? 4 : 8; }
static size_t vec_smem(int max_n, int max_nrhs) { return (size_t)max_n * (8 * vec_r(max_nrhs) + 4); }

bool getrs_vec_ok(int max_n, int max_nrhs) {
    return max_n > 0 && max_nrhs >= 1 && max_nrhs <= GV_MAX_NRHS && vec_smem(max_n, max_nrhs) <= 200 * 1024;
}

template <int R>
static void launch_r(int batch, size_t smem, const int *n, const int *nrhs, const double *const *A, const int *lda,
                     int *const *ipiv, double *const *B, const int *ldb, const int *mask, cudaStream_t s) {
    // always: the static tri tile counts against the default 48 KB as well
    smem_optin(getrs_vec_kernel<R>, smem);
    getrs_vec_kernel<R><<<batch, GV_THREADS, smem, s>>>(n, nrhs, A, lda, ipiv, B, ldb, mask);
}

void launch_getrs_vec(int batch, int max_n, int max_nrhs, const int *n, const int *nrhs, const double *const *A,
                      const int *lda, int *const *ipiv, double *const *B, const int *ldb, const int *mask,
                      cudaStream_t s) {
    const size_t smem = vec_smem(max_n, max_nrhs);
    KScope k(K_GETRS, s);
    switch (vec_r(max_nrhs)) {
        case 1: launch_r<1>(batch, smem, n, nrhs, A, lda, ipiv, B, ldb, mask, s); break;
        case 2: launch_r<2>(batch, smem, n, nrhs, A, lda, ipiv, B, ldb, mask, s); break;
        case 4: launch_r<4>(batch, smem, n, nrhs, A, lda, ipiv, B, ldb, mask, s); break;
        default: launch_r<8>(batch, smem, n, nrhs, A, lda, ipiv, B, ldb, mask, s); break;
    }
}

}  // namespace irr

// partial.cu -- argument validation of the partial front factorization
// (§III-A); the steps themselves are composed in api.cu from the
// getrf tiers, irrLASWP, irrTRSM and irrGEMM.
#include "irr_internal.cuh"

namespace irr {

__global__ void partial_validate_kernel(int batch, int max_n1, int max_n2, const int *n1, const int *n2,
                                        const int *ld11, const int *ld12, const int *ld21, const int *ld22,
                                        double *const *F11, double *const *F12, const double *const *F21,
                                        double *const *F22, int *const *ipiv, int *info) {
    const int i = blockIdx.x * blockDim.x + threadIdx.x;
    if (i >= batch) return;
    const int a = n1[i], b = n2[i];
    int e = 0;
    if (a < 0 || a > max_n1) e = -1;
    else if (b < 0 || b > max_n2) e = -2;
    else if (a > 0 && F11[i] == nullptr) e = -3;
    else if (ld11[i] < (a > 1 ? a : 1)) e = -4;
    else if (a > 0 && b > 0 && F12[i] == nullptr) e = -5;
    else if (ld12[i] < (a > 1 ? a : 1)) e = -6;
    else if (a > 0 && b > 0 && F21[i] == nullptr) e = -7;
    else if (ld21[i] < (b > 1 ? b : 1)) e = -8;
    else if (b > 0 && F22[i] == nullptr) e = -9;
    else if (ld22[i] < (b > 1 ? b : 1)) e = -10;
    else if (a > 0 && ipiv[i] == nullptr) e = -11;
    info[i] = e;
}

void launch_partial_validate(int batch, int max_n1, int max_n2, const int *n1, const int *n2, const int *ld11,
                             const int *ld12, const int *ld21, const int *ld22, double *const *F11,
                             double *const *F12, const double *const *F21, double *const *F22, int *const *ipiv,
                             int *info, cudaStream_t s) {
    KScope k(K_MISC, s);
    partial_validate_kernel<<<(batch + 255) / 256, 256, 0, s>>>(batch, max_n1, max_n2, n1, n2, ld11, ld12, ld21,
                                                               ld22, F11, F12, F21, F22, ipiv, info);
}

// irr_getrs argument check (LAPACK positions of the irr_getrs call)
__global__ void getrs_validate_kernel(int batch, int max_n, int max_nrhs, const int *n, const int *nrhs,
                                      const double *const *A, const int *lda, int *const *ipiv,
                                      double *const *B, const int *ldb, int *info) {
    // one warp per system: the scalar checks, then every pivot must name a row
    // in [k+1, n] (the solve kernels index shared memory with them)
    const int lane = threadIdx.x & 31;
    const int i = (blockIdx.x * blockDim.x + threadIdx.x) >> 5;
    if (i >= batch) return;
    const int a = n[i], b = nrhs[i];
    int e = 0;
    if (a < 0 || a > max_n) e = -5;
    else if (b < 0 || b > max_nrhs) e = -6;
    else if (a > 0 && A[i] == nullptr) e = -7;
    else if (lda[i] < (a > 1 ? a : 1)) e = -8;
    else if (a > 0 && ipiv[i] == nullptr) e = -9;
    else if (a > 0 && b > 0 && B[i] == nullptr) e = -10;
    else if (ldb[i] < (a > 1 ? a : 1)) e = -11;
    if (e == 0 && a > 0) {
        const int *p = ipiv[i];
        bool bad = false;
        for (int k = lane; k < a; k += 32) {
            const int v = p[k];
            bad |= v < k + 1 || v > a;
        }
        if (__any_sync(FULL, bad)) e = -9;
    }
    if (lane == 0) info[i] = e;
}

void launch_getrs_validate(int batch, int max_n, int max_nrhs, const int *n, const int *nrhs,
                           const double *const *A, const int *lda, int *const *ipiv, double *const *B,
                           const int *ldb, int *info, cudaStream_t s) {
    KScope k(K_MISC, s);
    getrs_validate_kernel<<<(batch + 7) / 8, 256, 0, s>>>(batch, max_n, max_nrhs, n, nrhs, A, lda, ipiv, B, ldb,
                                                         info);
}

// a6: per-matrix status words (info, FNV-1a of the pivot bytes), one thread
// per matrix (the pivot vectors are short; this is bookkeeping, not the path)
__global__ void status_words_kernel(int batch, const int *m, const int *n, int *const *ipiv, const int *info,
                                    unsigned *words) {
    const int i = blockIdx.x * blockDim.x + threadIdx.x;
    if (i >= batch) return;
    const int e = info[i];
    unsigned h = 2166136261u;
    if (e >= 0) {
        const int k = m[i] < n[i] ? m[i] : n[i];
        const int *p = ipiv[i];
        for (int t = 0; t < k; ++t) {
            const unsigned v = (unsigned)p[t];
#pragma unroll
            for (int b = 0; b < 4; ++b) {
                h ^= (v >> (8 * b)) & 0xffu;
                h *= 16777619u;
            }
        }
    } else {
        h = 0u;
    }
    words[2 * i] = (unsigned)e;
    words[2 * i + 1] = h;
}

void launch_status_words(int batch, const int *m, const int *n, int *const *ipiv, const int *info, unsigned *words,
                         cudaStream_t s) {
    KScope k(K_MISC, s);
    status_words_kernel<<<(batch + 255) / 256, 256, 0, s>>>(batch, m, n, ipiv, info, words);
}

}  // namespace irr

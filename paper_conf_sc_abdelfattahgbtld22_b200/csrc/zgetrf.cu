// zgetrf.cu -- irr_zgetrf: variable-size batched COMPLEX LU with partial
// pivoting (the sparse solver's A is in C^{N x N},
// PAPER.md L71 §III-A; the batch / DCWI interface of P:L121-133).
//
// Semantics follow LAPACK zgetf2 (DESIGN reading Q20): pivot = the smallest
// row maximising |Re| + |Im| (izamax), exact zero pivot -> info = first
// step, no interchange, no scaling; the multipliers are a_ik * (1 / a_kk)
// with 1 / a_kk = conj(a_kk) / |a_kk|^2 computed once per column (SURVEY
// reading Q6: the oracle divides, the tolerance absorbs the rounding; on
// the exact complex family every step is exact either way).
//
// One CTA per matrix (persistent, largest first from a device size sort):
// blocked right-looking LU with panels of ZNB columns:
//   panel   column by column: block arg-max of |Re| + |Im| (warp shuffles +
//           one smem round), the row interchange across all n columns, the
//           scaling, the rank-1 update of the panel's remaining columns;
//   U12     forward substitution with the unit L11 (staged in shared memory),
//           one thread per column, the column in registers;
//   A22    -= L21 U12 in 64 x 64 complex tiles: operands staged in shared
//           memory, 4 x 4 complex outputs per thread (4 DFMA per complex FMA).
// Matrices of up to ZSM_ELEMS complex elements are staged in shared memory
// for the whole factorization (read once, written once); larger ones are
// factored in place in global memory (L2-resident while their CTA works).
#include "irr_internal.cuh"
#include "sched.cuh"

namespace irr {

constexpr int ZT = 256;           // threads per CTA
constexpr int ZNB = 16;           // panel width (complex columns)
constexpr int ZTM = 64, ZTN = 64; // trailing-update tile (complex)
constexpr int ZSM_ELEMS = 4096;   // complex elements staged in shared memory (64 KB)
constexpr size_t Z_SMEM = (size_t)ZSM_ELEMS * 16 + (size_t)(ZNB * ZTM + ZNB * ZTN) * 16 + (size_t)ZNB * ZNB * 16;

__device__ __forceinline__ double2 zmul(double2 a, double2 b) {
    return make_double2(fma(a.x, b.x, -a.y * b.y), fma(a.x, b.y, a.y * b.x));
}
// c - a b
__device__ __forceinline__ double2 zfms(double2 c, double2 a, double2 b) {
    return make_double2(c.x - fma(a.x, b.x, -a.y * b.y), c.y - fma(a.x, b.y, a.y * b.x));
}

__global__ void zkey_kernel(ZArgs a, int *key) {
    const int i = blockIdx.x * blockDim.x + threadIdx.x;
    if (i >= a.batch) return;
    const double m = a.m[i] > 0 ? a.m[i] : 0, n = a.n[i] > 0 ? a.n[i] : 0;
    key[i] = (int)cbrt(m * n * (m < n ? m : n));
}

// block arg-max of cabs1 over rows [r0, m) of column c: (row, 1-based info of zero)
__device__ __forceinline__ int z_iamax(const double2 *A, long ld, int r0, int m, int c, unsigned long long *skey,
                                       int *srow) {
    const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
    unsigned long long bk = 0;
    int br = 0x7fffffff;
    for (int r = r0 + tid; r < m; r += ZT) {
        const double2 v = A[r + (size_t)c * ld];
        const unsigned long long k = (unsigned long long)__double_as_longlong(fabs(v.x) + fabs(v.y));
        if (br == 0x7fffffff || k > bk) { bk = k; br = r; }   // rows ascending: ties keep the smallest
    }
    unsigned long long wk;
    int wr;
    warp_argmax(br != 0x7fffffff, bk, br, wk, wr);
    if (lane == 0) { skey[warp] = wk; srow[warp] = wr; }
    __syncthreads();
    unsigned long long k = 0;
    int p = -1;
#pragma unroll
    for (int w = 0; w < ZT / 32; ++w) {
        const int rr = srow[w];
        if (rr < 0) continue;
        if (p < 0 || skey[w] > k || (skey[w] == k && rr < p)) { k = skey[w]; p = rr; }
    }
    __syncthreads();  // skey / srow are reused by the next column
    return p;
}

__global__ void __launch_bounds__(ZT) zgetrf_kernel(ZArgs a, int *queue, SlotList order) {
    extern __shared__ __align__(16) double z_smem[];
    double2 *sm_mat = reinterpret_cast<double2 *>(z_smem);
    double2 *sL = sm_mat + ZSM_ELEMS;   // [ZNB][ZTM]: L21 tile, k-major
    double2 *sU = sL + ZNB * ZTM;       // [ZNB][ZTN]: U12 tile
    double2 *sT = sU + ZNB * ZTN;       // L11 (ZNB x ZNB, column-major)
    __shared__ unsigned long long skey[ZT / 32];
    __shared__ int srow[ZT / 32];
    __shared__ int item_s;
    const int tid = threadIdx.x;
    const int count = order.count(a.batch);
    for (;;) {
        if (tid == 0) item_s = atomicAdd(queue, 1);
        __syncthreads();
        const int t = item_s;
        __syncthreads();
        if (t >= count) break;
        const int i = order.matrix(t);
        const int m = a.m[i], n = a.n[i];
        int e = 0;
        if (m < 0 || m > a.max_m) e = -1;
        else if (n < 0 || n > a.max_n) e = -2;
        else if (m > 0 && n > 0 && a.A[i] == nullptr) e = -3;
        else if (a.ld[i] < (m > 1 ? m : 1)) e = -4;
        else if (m > 0 && n > 0 && a.ipiv[i] == nullptr) e = -5;
        if (e || m == 0 || n == 0) {
            if (tid == 0) a.info[i] = e;
            continue;
        }
        const long gld = a.ld[i];
        double2 *G = reinterpret_cast<double2 *>(a.A[i]);
        int *ip = a.ipiv[i];
        // whole matrix in shared memory when it fits (generic pointers: the
        // code below runs on either)
        const bool staged = (long)m * n <= ZSM_ELEMS;
        double2 *A = staged ? sm_mat : G;
        const long ld = staged ? m : gld;
        if (staged) {
            for (int c = tid >> 5; c < n; c += ZT / 32)
                for (int r = tid & 31; r < m; r += 32) sm_mat[r + (size_t)c * m] = G[r + (size_t)c * gld];
            __syncthreads();
        }
        const int K = m < n ? m : n;
        int info = 0;
        for (int j = 0; j < K; j += ZNB) {
            const int ib = K - j < ZNB ? K - j : ZNB, c1 = j + ib;
            // ---- panel: columns [j, c1), rows [j, m)
            for (int k = j; k < c1; ++k) {
                const int p = z_iamax(A, ld, k, m, k, skey, srow);
                if (tid == 0) ip[k] = p + 1;
                const double2 pv = A[p + (size_t)k * ld];
                __syncthreads();  // every thread has the pivot before the interchange moves it
                const bool nz = pv.x != 0.0 || pv.y != 0.0;
                if (nz) {
                    if (p != k)
                        for (int c = tid; c < n; c += ZT) {
                            const double2 x = A[k + (size_t)c * ld];
                            A[k + (size_t)c * ld] = A[p + (size_t)c * ld];
                            A[p + (size_t)c * ld] = x;
                        }
                    __syncthreads();
                    const double den = pv.x * pv.x + pv.y * pv.y;
                    const double2 rc = make_double2(pv.x / den, -pv.y / den);
                    for (int r = k + 1 + tid; r < m; r += ZT) A[r + (size_t)k * ld] = zmul(A[r + (size_t)k * ld], rc);
                } else if (info == 0) {
                    info = k + 1;
                }
                __syncthreads();
                // rank-1 update of the panel's columns (k, c1)
                const int w = c1 - k - 1;
                if (w > 0)
                    for (int r = k + 1 + tid; r < m; r += ZT) {
                        const double2 l = A[r + (size_t)k * ld];
                        for (int c = k + 1; c < c1; ++c) A[r + (size_t)c * ld] = zfms(A[r + (size_t)c * ld], l, A[k + (size_t)c * ld]);
                    }
                __syncthreads();
            }
            if (c1 >= n) continue;
            // ---- U12 <- L11^-1 A12: L11 staged, one thread per column
            for (int e2 = tid; e2 < ib * ib; e2 += ZT) {
                const int r = e2 % ib, c = e2 / ib;
                sT[r + c * ZNB] = A[j + r + (size_t)(j + c) * ld];
            }
            __syncthreads();
            for (int c = c1 + tid; c < n; c += ZT) {
                double2 x[ZNB];
#pragma unroll
                for (int r = 0; r < ZNB; ++r) x[r] = r < ib ? A[j + r + (size_t)c * ld] : make_double2(0.0, 0.0);
#pragma unroll
                for (int s = 0; s < ZNB; ++s) {
#pragma unroll
                    for (int r = s + 1; r < ZNB; ++r)
                        if (r < ib) x[r] = zfms(x[r], sT[r + s * ZNB], x[s]);
                }
#pragma unroll
                for (int r = 0; r < ZNB; ++r)
                    if (r < ib) A[j + r + (size_t)c * ld] = x[r];
            }
            __syncthreads();
            if (c1 >= m) continue;
            // ---- A22 -= L21 U12 (K = ib), 64 x 64 complex tiles
            const int M2 = m - c1, N2 = n - c1;
            const int tx = tid & 15, ty = tid >> 4;
            for (int r0 = 0; r0 < M2; r0 += ZTM) {
                for (int e2 = tid; e2 < ZNB * ZTM; e2 += ZT) {
                    const int r = e2 % ZTM, s = e2 / ZTM;
                    sL[s * ZTM + r] = (r0 + r < M2 && s < ib) ? A[c1 + r0 + r + (size_t)(j + s) * ld]
                                                               : make_double2(0.0, 0.0);
                }
                for (int q0 = 0; q0 < N2; q0 += ZTN) {
                    for (int e2 = tid; e2 < ZNB * ZTN; e2 += ZT) {
                        const int s = e2 % ZNB, c = e2 / ZNB;
                        sU[s * ZTN + c] = (q0 + c < N2 && s < ib) ? A[j + s + (size_t)(c1 + q0 + c) * ld]
                                                                  : make_double2(0.0, 0.0);
                    }
                    __syncthreads();
                    double2 acc[4][4];
#pragma unroll
                    for (int u = 0; u < 4; ++u)
#pragma unroll
                        for (int v = 0; v < 4; ++v) acc[u][v] = make_double2(0.0, 0.0);
                    for (int s = 0; s < ib; ++s) {
                        double2 l[4], x[4];
#pragma unroll
                        for (int u = 0; u < 4; ++u) l[u] = sL[s * ZTM + tx + 16 * u];
#pragma unroll
                        for (int v = 0; v < 4; ++v) x[v] = sU[s * ZTN + ty + 16 * v];
#pragma unroll
                        for (int u = 0; u < 4; ++u)
#pragma unroll
                            for (int v = 0; v < 4; ++v) {
                                acc[u][v].x = fma(l[u].x, x[v].x, acc[u][v].x);
                                acc[u][v].x = fma(-l[u].y, x[v].y, acc[u][v].x);
                                acc[u][v].y = fma(l[u].x, x[v].y, acc[u][v].y);
                                acc[u][v].y = fma(l[u].y, x[v].x, acc[u][v].y);
                            }
                    }
#pragma unroll
                    for (int u = 0; u < 4; ++u) {
                        const int r = r0 + tx + 16 * u;
                        if (r >= M2) continue;
#pragma unroll
                        for (int v = 0; v < 4; ++v) {
                            const int c = q0 + ty + 16 * v;
                            if (c >= N2) continue;
                            double2 *dst = &A[c1 + r + (size_t)(c1 + c) * ld];
                            const double2 o = *dst;
                            *dst = make_double2(o.x - acc[u][v].x, o.y - acc[u][v].y);
                        }
                    }
                    __syncthreads();
                }
            }
        }
        if (staged) {
            __syncthreads();
            for (int c = tid >> 5; c < n; c += ZT / 32)
                for (int r = tid & 31; r < m; r += 32) G[r + (size_t)c * gld] = sm_mat[r + (size_t)c * m];
        }
        if (tid == 0) a.info[i] = info;
        __syncthreads();
    }
}

void launch_zgetrf(const ZArgs &a, int *counters, int *keys, int *sort_ws, cudaStream_t s) {
    cudaMemsetAsync(counters, 0, CNT_INTS * sizeof(int), s);
    {
        KScope k(K_MISC, s);
        zkey_kernel<<<(a.batch + 255) / 256, 256, 0, s>>>(a, keys);
    }
    launch_size_sort(keys, a.batch, sort_ws, s);
    SlotList order = sorted_slots(sort_ws, a.batch, -1);
    smem_optin(zgetrf_kernel, Z_SMEM);
    int grid = num_sms() * 2;
    if (grid > a.batch) grid = a.batch;
    KScope k(K_ZGETRF, s);
    zgetrf_kernel<<<grid, ZT, Z_SMEM, s>>>(a, counters + CNT_ZQ, order);
}

}  // namespace irr


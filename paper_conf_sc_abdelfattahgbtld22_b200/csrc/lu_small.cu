// lu_small.cu -- tier S: one warp per matrix, m, n <= 32, register resident
// (SURVEY §8(a) a2).
//
// Prior work handled <= 32x32 matrices by caching in shared memory with
// column-wise elimination; STRUMPACK's naive small kernel was
// launch bound.  Here the whole GEPP of one matrix runs in one warp:
//   lane r holds row r (n values in registers);
//   step k: warp arg-max of |a_rk| over the not-yet-pivotal rows with the
//   idamax tie rule (3 redux.sync), the row interchange is a relabelling of
//   lane positions (no data moves), the pivot row is broadcast through a
//   256-byte shared slot, scale and rank-1 update are register FMAs.
// Loads/stores are flat and fully coalesced (the matrix is staged through
// shared memory and transposed to rows there).  The warp-uniform size class
// (8 / 16 / 32 columns) keeps small matrices from paying for 32 columns.
#include "irr_internal.cuh"

namespace irr {

constexpr int S_WARPS = 4;

template <int NC>
__device__ __forceinline__ void lu_warp(double *__restrict__ gA, int m, int n, int ld, int *__restrict__ gipiv,
                                        int *__restrict__ ginfo, double *__restrict__ stage,
                                        double *__restrict__ prow, int lane) {
    const int total = m * n;
    // ---- coalesced load: global -> stage (packed column-major, ld_s = m)
    if (ld == m) {
        for (int e = lane; e < total; e += 32) stage[e] = gA[e];
    } else {
        for (int e = lane; e < total; e += 32) {
            int c = e / m, r = e - c * m;
            stage[e] = gA[r + (size_t)c * ld];
        }
    }
    __syncwarp();
    double a[NC];
#pragma unroll
    for (int c = 0; c < NC; ++c) a[c] = (lane < m && c < n) ? stage[lane + c * m] : 0.0;

    int pos = lane;      // current row position of the row held by this lane
    int my_piv = 0;      // ipiv[lane] (written by lane k at step k)
    int info = 0;
    const int K = m < n ? m : n;
    const bool valid = lane < m;
#pragma unroll
    for (int k = 0; k < NC; ++k) {
        if (k >= K) break;  // warp-uniform
        // ---- pivot search: max |a_.k| over positions >= k, tie -> smallest position
        const bool cand = valid && pos >= k;
        unsigned long long key;
        int pmin;
        warp_argmax(cand, dkey(fabs(a[k])), pos, key, pmin);
        const unsigned wmask = __ballot_sync(FULL, cand && pos == pmin);
        const int w = __ffs(wmask) - 1;
        if (lane == k) my_piv = pmin + 1;
        const double pv = __shfl_sync(FULL, a[k], w);
        // ---- interchange rows k and pmin: relabel positions only
        if (pos == k) pos = pmin;
        if (lane == w) pos = k;
        // ---- broadcast the pivot row (columns > k)
        if (lane == w) {
#pragma unroll
            for (int c = k + 1; c < NC; ++c) prow[c] = a[c];
        }
        __syncwarp();
        const bool below = valid && pos > k;
        if (pv != 0.0) {
            PivotScale sc(pv);
            if (below) a[k] = sc(a[k]);
        } else if (info == 0) {
            info = k + 1;  // exact zero pivot: no interchange (pmin == k), no scaling
        }
        if (below) {
            const double l = a[k];
#pragma unroll
            for (int c = k + 1; c < NC; ++c) a[c] = fma(-l, prow[c], a[c]);
        }
        __syncwarp();
    }
    // ---- write back: row held by this lane goes to its final position
    if (valid) {
#pragma unroll
        for (int c = 0; c < NC; ++c)
            if (c < n) stage[pos + c * m] = a[c];
    }
    __syncwarp();
    if (ld == m) {
        for (int e = lane; e < total; e += 32) gA[e] = stage[e];
    } else {
        for (int e = lane; e < total; e += 32) {
            int c = e / m, r = e - c * m;
            gA[r + (size_t)c * ld] = stage[e];
        }
    }
    if (lane < K) gipiv[lane] = my_piv;
    if (lane == 0) *ginfo = info;
    __syncwarp();  // stage is reused by the next matrix
}

__global__ void __launch_bounds__(32 * S_WARPS) lu_small_kernel(GetrfArgs a, const int *__restrict__ counters,
                                                                 const int *__restrict__ bins) {
    __shared__ double stage[S_WARPS][32 * 32];
    __shared__ double prow[S_WARPS][32];
    const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
    const int count = counters[CNT_BIN0 + BIN_S];
    const int *list = bins + (size_t)BIN_S * a.batch;
    for (int t = blockIdx.x * S_WARPS + warp; t < count; t += gridDim.x * S_WARPS) {
        const int i = list[t];
        const int m = a.m[i], n = a.n[i], ld = a.ld[i];
        if (n <= 8)
            lu_warp<8>(a.A[i], m, n, ld, a.ipiv[i], a.info + i, stage[warp], prow[warp], lane);
        else if (n <= 16)
            lu_warp<16>(a.A[i], m, n, ld, a.ipiv[i], a.info + i, stage[warp], prow[warp], lane);
        else
            lu_warp<32>(a.A[i], m, n, ld, a.ipiv[i], a.info + i, stage[warp], prow[warp], lane);
    }
}

void launch_lu_small(const GetrfArgs &a, const int *counters, const int *bins, cudaStream_t s) {
    // persistent grid: enough resident warps to cover HBM latency
    int grid = num_sms() * 8;
    int need = (a.batch + S_WARPS - 1) / S_WARPS;
    if (grid > need) grid = need;
    if (grid < 1) grid = 1;
    KScope k(K_LU_SMALL, s);
    lu_small_kernel<<<grid, 32 * S_WARPS, 0, s>>>(a, counters, bins);
}

}  // namespace irr

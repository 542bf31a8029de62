// lu_small.cu -- tier S: one warp per matrix, m, n <= 32, register resident
// (SURVEY §8(a) a2).
//
// Prior work handled <= 32x32 matrices by caching in shared memory with
// column-wise elimination; STRUMPACK's naive small kernel was
// launch bound.  Here the whole GEPP of one matrix runs in one warp:
//   * lane r holds row r in registers, SHIFTED so that a[0] is always the
//     current pivot column: the rank-1 update and the shift are one FMA per
//     register, a[c] <- a[c+1] - l * u[c+1], so every elimination step runs the
//     same code (a loop, not a 32x32 unrolled triangle -- the unrolled form
//     thrashed the instruction cache, ncu: 80% "no instruction" stalls);
//   * the step width W shrinks 32 -> 16 -> 8 -> 4 as the active columns do;
//   * pivot search: warp arg-max with the idamax tie rule (3 redux.sync);
//     the interchange relabels lane positions, only the already-final L
//     columns are swapped in shared memory (one lane per column);
//   * the pivot row is broadcast through a 256-byte shared slot (STS.128 /
//     LDS.128), U rows and L columns are written to the staged output as soon
//     as they are final.
// Loads are cp.async (the next matrix is in flight while the current one is
// factored); stores are flat and fully coalesced.
#include "irr_internal.cuh"

namespace irr {

constexpr int S_WARPS = 4;
constexpr int S_STAGE = 1024;  // doubles per stage buffer (32 x 32)

template <int NC, int W>
__device__ __forceinline__ void s_step(double (&a)[NC], int &k, int &pos, int &my_piv, int &info, int m, int n,
                                       int lane, double *__restrict__ st, double *__restrict__ prow) {
    const bool valid = lane < m;
    const bool cand = valid && pos >= k;
    unsigned long long key;
    int pmin;
    warp_argmax(cand, dkey(fabs(a[0])), pos, key, pmin);
    const unsigned wmask = __ballot_sync(FULL, cand && pos == pmin);
    const int w = __ffs(wmask) - 1;
    if (lane == k) my_piv = pmin + 1;
    if (lane == w) {
#pragma unroll
        for (int c = 0; c < W; c += 2) *reinterpret_cast<double2 *>(prow + c) = make_double2(a[c], a[c + 1]);
    }
    __syncwarp();
    const double pv = prow[0];
    // interchange the final L columns (< k) of positions k and pmin
    if (pmin != k && lane < k) {
        const double x = st[k + lane * m], y = st[pmin + lane * m];
        st[k + lane * m] = y;
        st[pmin + lane * m] = x;
    }
    // U row k is final: columns k .. n-1 (n - k <= W <= 32)
    if (lane < n - k) st[k + (k + lane) * m] = prow[lane];
    if (pos == k) pos = pmin;
    if (lane == w) pos = k;
    const bool below = valid && pos > k;
    double l = a[0];
    if (pv != 0.0) {
        if (fabs(pv) >= DBL_MIN) l = l * (1.0 / pv);
        else l = l / pv;
    } else if (info == 0) {
        info = k + 1;  // exact zero pivot: pmin == k (no interchange), no scaling
    }
    if (below) st[pos + k * m] = l;
    double u[W];
#pragma unroll
    for (int c = 0; c < W; c += 2) {
        const double2 v = *reinterpret_cast<const double2 *>(prow + c);
        u[c] = v.x;
        u[c + 1] = v.y;
    }
#pragma unroll
    for (int c = 0; c + 1 < W; ++c) a[c] = fma(-l, u[c + 1], a[c + 1]);
    a[W - 1] = 0.0;
    __syncwarp();
    ++k;
}

template <int NC>
__device__ __forceinline__ void lu_warp(double *__restrict__ gA, int m, int n, int ld, int *__restrict__ gipiv,
                                        int *__restrict__ ginfo, double *__restrict__ st,
                                        double *__restrict__ prow, int lane) {
    const int total = m * n;
    double a[NC];
#pragma unroll
    for (int c = 0; c < NC; ++c) a[c] = (lane < m && c < n) ? st[lane + c * m] : 0.0;
    __syncwarp();
    int pos = lane, my_piv = 0, info = 0, k = 0;
    const int K = m < n ? m : n;
    if (NC >= 32)
        while (k < K && n - k > 16) s_step<NC, (NC >= 32 ? 32 : NC)>(a, k, pos, my_piv, info, m, n, lane, st, prow);
    if (NC >= 16)
        while (k < K && n - k > 8) s_step<NC, (NC >= 16 ? 16 : NC)>(a, k, pos, my_piv, info, m, n, lane, st, prow);
    while (k < K && n - k > 4) s_step<NC, (NC >= 8 ? 8 : NC)>(a, k, pos, my_piv, info, m, n, lane, st, prow);
    while (k < K) s_step<NC, 4>(a, k, pos, my_piv, info, m, n, lane, st, prow);
    __syncwarp();
    if (ld == m) {
        for (int e = lane; e < total; e += 32) gA[e] = st[e];
    } else {
        for (int e = lane; e < total; e += 32) {
            int c = e / m, r = e - c * m;
            gA[r + (size_t)c * ld] = st[e];
        }
    }
    if (lane < K) gipiv[lane] = my_piv;
    if (lane == 0) *ginfo = info;
    __syncwarp();  // the stage buffer is refilled by the next prefetch
}

// Each warp walks its share of the tier-S list with a two-deep pipeline: the
// next matrix is in flight (cp.async into the other stage buffer) while the
// current one is factored.
__global__ void __launch_bounds__(32 * S_WARPS) lu_small_kernel(GetrfArgs a, const int *__restrict__ counters,
                                                                 const int *__restrict__ bins) {
    extern __shared__ __align__(16) double s_small[];
    const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
    double *stage0 = s_small + (size_t)warp * (2 * S_STAGE + 32);
    double *prow = stage0 + 2 * S_STAGE;
    const int count = counters[CNT_BIN0 + BIN_S];
    const int *list = bins + (size_t)BIN_S * a.batch;
    const int stride = gridDim.x * S_WARPS;
    int t = blockIdx.x * S_WARPS + warp;
    if (t >= count) return;
    int i = list[t];
    int m = a.m[i], n = a.n[i], ld = a.ld[i];
    double *gA = a.A[i];
    stage_block_async(stage0, m, gA, ld, m, n, lane, 32);
    cp_async_commit();
    int cur = 0;
    while (true) {
        const int tn = t + stride;
        int i2 = 0, m2 = 0, n2 = 0, ld2 = 0;
        double *gA2 = nullptr;
        if (tn < count) {
            i2 = list[tn];
            m2 = a.m[i2]; n2 = a.n[i2]; ld2 = a.ld[i2];
            gA2 = a.A[i2];
            stage_block_async(stage0 + (cur ^ 1) * S_STAGE, m2, gA2, ld2, m2, n2, lane, 32);
        }
        cp_async_commit();
        cp_async_wait<1>();
        __syncwarp();
        double *st = stage0 + cur * S_STAGE;
        if (n <= 8)
            lu_warp<8>(gA, m, n, ld, a.ipiv[i], a.info + i, st, prow, lane);
        else if (n <= 16)
            lu_warp<16>(gA, m, n, ld, a.ipiv[i], a.info + i, st, prow, lane);
        else
            lu_warp<32>(gA, m, n, ld, a.ipiv[i], a.info + i, st, prow, lane);
        if (tn >= count) break;
        t = tn; i = i2; m = m2; n = n2; ld = ld2; gA = gA2;
        cur ^= 1;
    }
    cp_async_wait<0>();
}

void launch_lu_small(const GetrfArgs &a, const int *counters, const int *bins, cudaStream_t s) {
    const size_t smem = (size_t)S_WARPS * (2 * S_STAGE + 32) * sizeof(double);
    static size_t attr = 0;
    if (smem > attr) {
        cudaFuncSetAttribute(lu_small_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
        attr = smem;
    }
    int grid = num_sms() * 3;  // 3 x 66 KB per SM: 12 warps / SM, 2 matrices in flight per warp
    int need = (a.batch + S_WARPS - 1) / S_WARPS;
    if (grid > need) grid = need;
    if (grid < 1) grid = 1;
    KScope k(K_LU_SMALL, s);
    lu_small_kernel<<<grid, 32 * S_WARPS, smem, s>>>(a, counters, bins);
}

}  // namespace irr

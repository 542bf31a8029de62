// classify.cu -- the device-side DCWI / size-binning step.
//
// DCWI: "each developed kernel internally infers the actual
// sizes ... If no workload is detected, the corresponding GPU threads perform
// no work at all."  Here one pass over the local dims validates every matrix
// (LAPACK-style info < 0, the matrix is then skipped), and appends it to the
// compacted list of its size class.  Later kernels loop over those device-side
// lists with persistent grids, so no per-matrix information ever crosses to
// the host (pointer/size arithmetic on the host is what the
// expanded interface avoids).
#include "irr_internal.cuh"

namespace irr {

__global__ void __launch_bounds__(256) classify_kernel(GetrfArgs a, int *counters, int *bins, int keep_neg_info,
                                                       int tier_s, int tier_m_max, int l1) {
    const int i = blockIdx.x * blockDim.x + threadIdx.x;
    const int lane = threadIdx.x & 31;
    int bin = -1;
    if (i < a.batch) {
        const int mi = a.m[i], ni = a.n[i];
        int e = 0;
        if (keep_neg_info && a.info[i] < 0) e = a.info[i];
        else if (mi < 0 || mi > a.max_m) e = -1;
        else if (ni < 0 || ni > a.max_n) e = -2;
        else if (mi > 0 && ni > 0 && a.A[i] == nullptr) e = -3;
        else if (a.ld[i] < (mi > 1 ? mi : 1)) e = -4;
        else if (mi > 0 && ni > 0 && a.ipiv[i] == nullptr) e = -5;
        a.info[i] = e;
        if (e == 0 && mi > 0 && ni > 0) {
            const long long el = (long long)mid_lds(mi) * ni;
            if (tier_s >= 2 && mi <= 8 && ni <= 8) bin = BIN_S8G;  // four matrices per warp
            else if (tier_s >= 2 && mi <= 16 && ni <= 16) bin = BIN_S16G;  // two per warp
            else if (tier_s && mi <= 32 && ni <= 32)
                bin = ni <= 8 ? BIN_S8 : (ni <= 16 ? BIN_S16 : ((tier_s >= 2 && ni <= 24) ? BIN_S24 : BIN_S));
            else if (el <= M1_ELEMS && el <= tier_m_max) bin = BIN_M1;
            else if (el <= M2_ELEMS && el <= tier_m_max) bin = BIN_M2;
            else if (el <= tier_m_max) bin = BIN_M3;
            else if (l1 && mi <= l1) bin = mi <= L1_MAX_ROWS ? BIN_L1 : BIN_L1T;  // l1 = max rows of the CTA-per-matrix tier
            else bin = BIN_L;
        }
    }
    // warp-aggregated append to the bin lists: lanes of equal bin found with
    // one match, one atomic per distinct bin of the warp (leader lane)
    const unsigned mask = __match_any_sync(FULL, bin);
    const int leader = __ffs(mask) - 1;
    int base = 0;
    if (lane == leader && bin >= 0) base = atomicAdd(&counters[CNT_BIN0 + bin], __popc(mask));
    base = __shfl_sync(FULL, base, leader);
    if (bin >= 0) bins[(size_t)bin * a.batch + base + __popc(mask & ((1u << lane) - 1))] = i;
}

void launch_classify(const GetrfArgs &a, int *counters, int *bins, int keep_neg_info, cudaStream_t s) {
    const Tuning &t = tuning();
    int grid = (a.batch + 255) / 256;
    KScope k(K_CLASSIFY, s);
    classify_kernel<<<grid, 256, 0, s>>>(a, counters, bins, keep_neg_info, t.tier_s, t.tier_m_max, t.l1 ? t.l1_rows : 0);
}

// max over the batch of the local dims (only when the caller passes required
// dims <= 0: the host then reads them back -- the one documented sync)
__global__ void max_dims_kernel(int batch, const int *m, const int *n, int *counters) {
    int mm = 0, nn = 0;
    for (int i = blockIdx.x * blockDim.x + threadIdx.x; i < batch; i += gridDim.x * blockDim.x) {
        mm = max(mm, m[i]);
        nn = max(nn, n[i]);
    }
    mm = __reduce_max_sync(FULL, (unsigned)max(mm, 0));
    nn = __reduce_max_sync(FULL, (unsigned)max(nn, 0));
    if ((threadIdx.x & 31) == 0) {
        atomicMax(&counters[CNT_MAXM], mm);
        atomicMax(&counters[CNT_MAXN], nn);
    }
}

void launch_max_dims(int batch, const int *m, const int *n, int *counters, cudaStream_t s) {
    int grid = (batch + 255) / 256;
    if (grid > 1024) grid = 1024;
    if (grid < 1) grid = 1;
    KScope k(K_MISC, s);
    max_dims_kernel<<<grid, 256, 0, s>>>(batch, m, n, counters);
}

}  // namespace irr

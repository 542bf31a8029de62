// lu_small.cu -- tier S: one warp per matrix, m, n <= 32, register resident
// (SURVEY §8(a) a2).
//
// Prior work handled <= 32x32 matrices by caching in shared memory with
// column-wise elimination; STRUMPACK's naive small kernel was
// launch bound.  Here the whole GEPP of one matrix runs in one warp
// and the matrix is read once and written once (HBM-bound, AI <= 1.33):
//   * lane r holds row r in registers, SHIFTED so that a[0] is always the
//     current pivot column: the rank-1 update and the shift are one FMA per
//     register, a[c] <- a[c+1] - l * u[c+1], so every elimination step runs the
//     same code; the step width W shrinks 32 -> 24 -> 16 -> 12 -> 8 -> 4
//     with the active columns;
//   * rows never move.  `pos` is the row's current position; an interchange
//     is a relabelling (the winner lane takes position k, the row at k takes
//     the winner's old position).  So nothing is swapped during the
//     factorization: the multiplier a lane computes at step k goes to
//     Lb[k][lane], the pivot row published at step k IS row k of U (Ub, rows
//     packed by decreasing length), and at the end every lane writes its row
//     once, at its final position -- for each column the warp's stores cover
//     exactly that column, so they stay coalesced;
//   * pivot search (idamax, ties -> smallest position): one
//     redux.max on the high word of |a| + a ballot; only when two lanes share
//     that high word does the full 64-bit compare + min-position run;
//   * the next warp's matrix is prefetched into L2 while this one is factored.
// Instruction count per matrix was the bound of the previous form (ncu: 2,625
// warp instructions per matrix of C1big, IPC 1.6 at 12 warps/SM); this form
// drops the per-step output bookkeeping and the smem input stage, and runs 16
// warps per SM.
#include "irr_internal.cuh"

namespace irr {

constexpr int S_WARPS = 4;
#ifndef IRR_S_PF
#define IRR_S_PF 1  // L2 prefetch distance of the warp-per-matrix kernels (items ahead)
#endif

// Width classes n <= 8 / 16 / 32 are separate bins and separate kernels
// (classify.cu), so the narrow ones run at their own register and
// shared-memory budgets: more resident warps to hide the per-step latency
// chain (redux -> ballot -> shfl -> publish -> LDS -> DMUL -> DFMA).
template <int NC>
struct SmallCfg;
template <>
struct SmallCfg<32> { static constexpr int ctas = 4, bin = BIN_S; };    // 128 regs, 16 warps / SM
#ifndef IRR_S24_CTAS
#define IRR_S24_CTAS 5
#endif
template <>
struct SmallCfg<24> { static constexpr int ctas = IRR_S24_CTAS, bin = BIN_S24; };  // 96 regs, 20 warps / SM (tier_s = 2)
template <>
struct SmallCfg<16> { static constexpr int ctas = 6, bin = BIN_S16; };  // 80 regs, 24 warps / SM
template <>
struct SmallCfg<8> { static constexpr int ctas = 8, bin = BIN_S8; };    // 64 regs, 32 warps / SM

// U rows are packed in step order, row k taking exactly its step width W(k)
// (the class of n - k: 32 / 24 / 16 / 12 / 8 / 4), so a step publishes and
// reads its full W-wide pair stores / loads without predicates and no step
// touches another row's slots.  Capacity = the widths summed at n = NC.
template <int NC>
__host__ __device__ constexpr int s_width(int rem) {
    return (NC >= 32 && rem > 28) ? 32 : (NC >= 32 && rem > 24) ? 28 : (NC >= 24 && rem > 20) ? 24
         : (NC >= 24 && rem > 16) ? 20 : (NC >= 16 && rem > 12) ? 16
         : (NC >= 16 && rem > 8) ? 12 : (rem > 4) ? (NC >= 8 ? 8 : NC) : 4;
}
template <int NC>
__host__ __device__ constexpr int s_ucap() {
    int t = 0;
    for (int k = 0; k < NC; ++k) t += s_width<NC>(NC - k);
    return t;
}

template <int NC>
struct __align__(16) SmallWarpSmem {  // 16-byte multiple: U rows take double2 stores in every warp's slot
    double L[NC * 32];             // L[k*32 + lane]: multiplier of the row held by `lane` at step k
    double U[s_ucap<NC>()];        // row k of U at urow[k], W(k) slots
    double rcp[2];                 // reciprocal of the pivot of step k in rcp[k & 1] (0: divide)
    int urow[NC];                  // offset of U row k
};
static_assert(sizeof(SmallWarpSmem<32>) % 16 == 0 && sizeof(SmallWarpSmem<24>) % 16 == 0 &&
                  sizeof(SmallWarpSmem<16>) % 16 == 0 && sizeof(SmallWarpSmem<8>) % 16 == 0,
              "per-warp slots must stay 16-byte aligned");
static_assert(s_ucap<32>() == 576 && s_ucap<24>() == 336 && s_ucap<16>() == 160 && s_ucap<8>() == 48,
              "packed U capacity");

template <int NC, int W>
__device__ __forceinline__ void s_step(double (&a)[NC], int &k, int &pos, int &my_piv, int &info, bool valid,
                                       int lane, int &uo, SmallWarpSmem<NC> &sm) {
    const bool cand = valid && pos >= k;
    // every lane's reciprocal of its own candidate, off the critical path of
    // the pivot search; the winner publishes its one
    const double myr = fast_rcp(a[0]);
    // ---- arg-max of |a[0]| over the candidates
    const unsigned long long key = (unsigned long long)__double_as_longlong(fabs(a[0]));
    const unsigned hi = cand ? (unsigned)(key >> 32) : 0u;
    const unsigned mhi = __reduce_max_sync(FULL, hi);
    const bool e1 = cand && hi == mhi;
    unsigned wm = __ballot_sync(FULL, e1);
    if (wm & (wm - 1)) {  // several lanes share the high word (rare): exact compare, then smallest position
        const unsigned mlo = __reduce_max_sync(FULL, e1 ? (unsigned)key : 0u);
        const bool e2 = e1 && (unsigned)key == mlo;
        const unsigned pm = __reduce_min_sync(FULL, e2 ? (unsigned)pos : 0xffffffffu);
        wm = __ballot_sync(FULL, e2 && pos == (int)pm);
    }
    const int w = __ffs(wm) - 1;
    const int pmin = __shfl_sync(FULL, pos, w);
    // ---- the pivot row is row k of U: publish it where the output reads it
    double *urow = sm.U + uo;
    if (lane == w) {
#pragma unroll
        for (int c = 0; c < W; c += 2) *reinterpret_cast<double2 *>(urow + c) = make_double2(a[c], a[c + 1]);
        sm.rcp[k & 1] = myr;
    }
    if (lane == 0) sm.urow[k] = uo;
    uo += W;
    if (lane == k) my_piv = pmin + 1;
    __syncwarp();
    const double pv = urow[0];
    const double rc = sm.rcp[k & 1];
    // ---- interchange = relabel positions
    if (pos == k) pos = pmin;
    if (lane == w) pos = k;
    const bool below = valid && pos > k;
    // common case branch-free (pv and rc are loaded together, the multiply
    // does not wait behind a branch on pv); divide / zero pivot are the rare paths
    double l = a[0] * rc;
    if (rc == 0.0) {
        if (pv != 0.0) l = a[0] / pv;  // |pv| < DBL_MIN or 1/pv subnormal (LAPACK divides below sfmin)
        else {
            l = a[0];
            if (info == 0) info = k + 1;  // exact zero pivot: every candidate is 0, pmin == k, no scaling
        }
    }
    if (below) sm.L[k * 32 + lane] = l;
    // ---- rank-1 update fused with the shift, u streamed in 16-byte loads
    constexpr int CH = W < 4 ? W : 4;
#pragma unroll
    for (int e0 = 0; e0 < W; e0 += CH) {
        double uu[CH];
#pragma unroll
        for (int q = 0; q < CH; q += 2) {
            const double2 v = *reinterpret_cast<const double2 *>(urow + e0 + q);
            uu[q] = v.x;
            uu[q + 1] = v.y;
        }
#pragma unroll
        for (int q = 0; q < CH; ++q)
            if (e0 + q >= 1) a[e0 + q - 1] = fma(-l, uu[q], a[e0 + q]);
    }
    a[W - 1] = 0.0;
    // no trailing warp barrier: the next step writes row k+1 (its own W
    // slots after row k's) and rcp[(k+1) & 1], neither of which this step reads
    ++k;
}

template <int NC>
__device__ __forceinline__ void lu_warp(double *__restrict__ gA, int m, int n, int ld, int *__restrict__ gipiv,
                                        int *__restrict__ ginfo, SmallWarpSmem<NC> &sm, int lane) {
    const bool valid = lane < m;
    double a[NC];
    const double *gr = gA + lane;
#pragma unroll
    for (int c = 0; c < NC; ++c) {
        a[c] = (valid && c < n) ? *gr : 0.0;
        gr += ld;
    }
    int pos = lane, my_piv = 0, info = 0, k = 0, uo = 0;
    const int K = m < n ? m : n;
    // active width W >= n - k in steps of 32 / 28 / 24 / 20 / 16 / 12 / 8 / 4 (the
    // FMAs, pivot-row loads and publish stores of a step scale with W)
    if (NC >= 32) {
        while (k < K && n - k > 28) s_step<NC, (NC >= 32 ? 32 : NC)>(a, k, pos, my_piv, info, valid, lane, uo, sm);
        while (k < K && n - k > 24) s_step<NC, (NC >= 32 ? 28 : NC)>(a, k, pos, my_piv, info, valid, lane, uo, sm);
    }
    if (NC >= 24) {
        while (k < K && n - k > 20) s_step<NC, (NC >= 24 ? 24 : NC)>(a, k, pos, my_piv, info, valid, lane, uo, sm);
        while (k < K && n - k > 16) s_step<NC, (NC >= 24 ? 20 : NC)>(a, k, pos, my_piv, info, valid, lane, uo, sm);
    }
    if (NC >= 16) {
        while (k < K && n - k > 12) s_step<NC, (NC >= 16 ? 16 : NC)>(a, k, pos, my_piv, info, valid, lane, uo, sm);
        while (k < K && n - k > 8) s_step<NC, (NC >= 16 ? 12 : NC)>(a, k, pos, my_piv, info, valid, lane, uo, sm);
    }
    while (k < K && n - k > 4) s_step<NC, (NC >= 8 ? 8 : NC)>(a, k, pos, my_piv, info, valid, lane, uo, sm);
    while (k < K) s_step<NC, 4>(a, k, pos, my_piv, info, valid, lane, uo, sm);
    __syncwarp();  // L / U rows from every lane are complete
    // ---- write every row once, at its final position p: L(p, c) for c < p,
    //      U(p, c) for c >= p (rows p >= K are pure L rows)
    if (valid) {
        double *go = gA + pos;
        const double *ur = sm.U + sm.urow[pos < K ? pos : 0] - pos;
        for (int c = 0; c < n; ++c) {
            double v;
            if (c < pos) v = sm.L[c * 32 + lane];
            else v = ur[c];
            go[(size_t)c * ld] = v;
        }
    }
    if (lane < K) gipiv[lane] = my_piv;
    if (lane == 0) *ginfo = info;
    __syncwarp();  // sm is rewritten by the next matrix
}

// ------------------------------------------------------------------ grouped
// Matrices with m, n <= GS (GS = 8 or 16): G = 32 / GS matrices per warp, one
// per lane group of GS lanes (lane = group * GS + row).  Same row-relabel
// shift form as lu_warp, but every warp instruction of a step now serves G
// matrices: the publish, the pivot-row loads, the multiplier stores and the
// FMAs are shared; only the pivot search is per group (G high-word reduxes,
// one ballot split by group).  The step loop runs to the largest K of the
// warp's matrices and the width class follows their largest n; a group whose
// matrix has no step k left sits the step out (no publish, no info, no L).
template <int GS>
struct __align__(16) GroupWarpSmem {
    static constexpr int G = 32 / GS;
    double L[GS * 32];               // L[k*32 + lane]
    double U[G][s_ucap<GS>()];       // per group: row k of U at urow[k], W(k) slots
    double rcp[G][2];                // per group: reciprocal of the pivot of step k in rcp[g][k & 1]
    int urow[GS];                    // warp-uniform packed offsets
};
static_assert(sizeof(GroupWarpSmem<8>) % 16 == 0 && sizeof(GroupWarpSmem<16>) % 16 == 0,
              "per-warp slots must stay 16-byte aligned");

template <int GS, int W>
__device__ __forceinline__ void g_step(double (&a)[GS], int k, int &pos, int &my_piv, int &info, bool valid,
                                       bool act, int lane, int uo, GroupWarpSmem<GS> &sm) {
    constexpr int G = 32 / GS;
    const int g = lane / GS, glane = lane & (GS - 1);
    const bool cand = valid && act && pos >= k;
    const double myr = fast_rcp(a[0]);
    // ---- per-group arg-max of |a[0]|: G reduxes on the high word, one ballot
    const unsigned long long key = (unsigned long long)__double_as_longlong(fabs(a[0]));
    const unsigned hi = cand ? (unsigned)(key >> 32) : 0u;
    unsigned mhi = 0;
#pragma unroll
    for (int q = 0; q < G; ++q) {
        const unsigned r = __reduce_max_sync(FULL, g == q ? hi : 0u);
        if (g == q) mhi = r;
    }
    const bool e1 = cand && hi == mhi;
    constexpr unsigned GM = GS == 32 ? 0xffffffffu : ((1u << GS) - 1u);
    unsigned gm = (__ballot_sync(FULL, e1) >> (g * GS)) & GM;
    if (__any_sync(FULL, (gm & (gm - 1)) != 0)) {  // a high-word tie in some group (rare)
        unsigned mlo = 0;
#pragma unroll
        for (int q = 0; q < G; ++q) {
            const unsigned r = __reduce_max_sync(FULL, (g == q && e1) ? (unsigned)key : 0u);
            if (g == q) mlo = r;
        }
        const bool e2 = e1 && (unsigned)key == mlo;
        unsigned pm = 0xffffffffu;
#pragma unroll
        for (int q = 0; q < G; ++q) {
            const unsigned r = __reduce_min_sync(FULL, (g == q && e2) ? (unsigned)pos : 0xffffffffu);
            if (g == q) pm = r;
        }
        gm = (__ballot_sync(FULL, e2 && pos == (int)pm) >> (g * GS)) & GM;
    }
    const int w = gm ? g * GS + __ffs(gm) - 1 : lane;  // winner lane of this group
    const int pmin = __shfl_sync(FULL, pos, w);
    // ---- publish the pivot rows (one lane per group)
    double *urow = sm.U[g] + uo;
    if (gm && lane == w) {
#pragma unroll
        for (int c = 0; c < W; c += 2) *reinterpret_cast<double2 *>(urow + c) = make_double2(a[c], a[c + 1]);
        sm.rcp[g][k & 1] = myr;
    }
    if (lane == 0) sm.urow[k] = uo;
    if (act && glane == k) my_piv = pmin + 1;
    __syncwarp();
    const double pv = urow[0];
    const double rc = sm.rcp[g][k & 1];
    if (act) {
        if (pos == k) pos = pmin;
        if (lane == w) pos = k;
    }
    const bool below = valid && act && pos > k;
    double l = a[0] * rc;
    if (rc == 0.0) {
        if (pv != 0.0) l = a[0] / pv;
        else {
            l = a[0];
            if (act && info == 0) info = k + 1;
        }
    }
    if (below) sm.L[k * 32 + lane] = l;
    constexpr int CH = W < 4 ? W : 4;
#pragma unroll
    for (int e0 = 0; e0 < W; e0 += CH) {
        double uu[CH];
#pragma unroll
        for (int q = 0; q < CH; q += 2) {
            const double2 v = *reinterpret_cast<const double2 *>(urow + e0 + q);
            uu[q] = v.x;
            uu[q + 1] = v.y;
        }
#pragma unroll
        for (int q = 0; q < CH; ++q)
            if (e0 + q >= 1) a[e0 + q - 1] = fma(-l, uu[q], a[e0 + q]);
    }
    a[W - 1] = 0.0;
    (void)glane;
}

template <int GS>
constexpr int group_ctas() { return GS == 8 ? 8 : 6; }  // 64 / 80 registers

template <int GS>
__global__ void __launch_bounds__(32 * S_WARPS, group_ctas<GS>()) lu_group_kernel(GetrfArgs a,
                                                                             const int *__restrict__ counters,
                                                                             const int *__restrict__ bins, int bin) {
    constexpr int G = 32 / GS;
    extern __shared__ __align__(16) double s_small[];
    const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
    const int g = lane / GS, glane = lane & (GS - 1);
    GroupWarpSmem<GS> &sm = reinterpret_cast<GroupWarpSmem<GS> *>(s_small)[warp];
    const int count = counters[CNT_BIN0 + bin];
    const int *list = bins + (size_t)bin * a.batch;
    const int items = (count + G - 1) / G;
    const int stride = gridDim.x * S_WARPS;
    for (int t = blockIdx.x * S_WARPS + warp; t < items; t += stride) {
        const int slot = t * G + g;
        int m = 0, n = 0, ld = 1, i = -1;
        if (slot < count) {
            i = list[slot];
            m = a.m[i];
            n = a.n[i];
            ld = a.ld[i];
        }
        // next item of this warp into L2, one lane group per matrix
        const int sn = (t + stride) * G + g;
        if (t + stride < items && sn < count) {
            const int i2 = list[sn];
            const char *p2 = reinterpret_cast<const char *>(a.A[i2]);
            const long bytes = ((long)(a.n[i2] - 1) * a.ld[i2] + a.m[i2]) * 8;
            for (long o = (long)glane * 128; o < bytes; o += GS * 128)
                asm volatile("prefetch.global.L2 [%0];" ::"l"(p2 + o));
        }
        const bool valid = glane < m;
        double a_[GS];
        {
            const double *gr = i >= 0 ? a.A[i] + glane : nullptr;
#pragma unroll
            for (int c = 0; c < GS; ++c) {
                a_[c] = (valid && c < n) ? gr[(size_t)c * ld] : 0.0;
            }
        }
        const int K = m < n ? m : n;
        const int Kmax = (int)__reduce_max_sync(FULL, (unsigned)K);
        const int nmax = (int)__reduce_max_sync(FULL, (unsigned)n);
        int pos = glane, my_piv = 0, info = 0, k = 0, uo = 0;
        if (GS >= 16) {
            for (; k < Kmax && nmax - k > 12; ++k, uo += 16)
                g_step<GS, 16>(a_, k, pos, my_piv, info, valid, k < K, lane, uo, sm);
            for (; k < Kmax && nmax - k > 8; ++k, uo += 12)
                g_step<GS, 12>(a_, k, pos, my_piv, info, valid, k < K, lane, uo, sm);
        }
        for (; k < Kmax && nmax - k > 4; ++k, uo += 8) g_step<GS, 8>(a_, k, pos, my_piv, info, valid, k < K, lane, uo, sm);
        for (; k < Kmax; ++k, uo += 4) g_step<GS, 4>(a_, k, pos, my_piv, info, valid, k < K, lane, uo, sm);
        __syncwarp();
        if (valid) {
            double *go = a.A[i] + pos;
            const double *ur = sm.U[g] + sm.urow[pos < K ? pos : 0] - pos;
            for (int c = 0; c < n; ++c) {
                double v;
                if (c < pos) v = sm.L[c * 32 + lane];
                else v = ur[c];
                go[(size_t)c * ld] = v;
            }
        }
        if (i >= 0) {
            if (glane < K) a.ipiv[i][glane] = my_piv;
            if (glane == 0) a.info[i] = info;
        }
        __syncwarp();
    }
}

template <int GS>
static void launch_group(const GetrfArgs &a, const int *counters, const int *bins, int bin, cudaStream_t s) {
    const size_t smem = (size_t)S_WARPS * sizeof(GroupWarpSmem<GS>);
    smem_optin(lu_group_kernel<GS>, smem);
    constexpr int G = 32 / GS;
    int grid = num_sms() * group_ctas<GS>();
    int need = (a.batch + S_WARPS * G - 1) / (S_WARPS * G);
    if (grid > need) grid = need;
    if (grid < 1) grid = 1;
    KScope k(K_LU_SMALL, s);
    lu_group_kernel<GS><<<grid, 32 * S_WARPS, smem, s>>>(a, counters, bins, bin);
}

// Each warp walks its share of the width class's list (static stride); the
// next matrix of the warp is prefetched into L2 before the current one is
// loaded.
template <int NC>
__global__ void __launch_bounds__(32 * S_WARPS, SmallCfg<NC>::ctas) lu_small_kernel(GetrfArgs a,
                                                                                    const int *__restrict__ counters,
                                                                                    const int *__restrict__ bins) {
    extern __shared__ __align__(16) double s_small[];
    const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
    SmallWarpSmem<NC> &sm = reinterpret_cast<SmallWarpSmem<NC> *>(s_small)[warp];
    const int count = counters[CNT_BIN0 + SmallCfg<NC>::bin];
    const int *list = bins + (size_t)SmallCfg<NC>::bin * a.batch;
    const int stride = gridDim.x * S_WARPS;
    for (int t = blockIdx.x * S_WARPS + warp; t < count; t += stride) {
        const int i = list[t];
        const int m = a.m[i], n = a.n[i], ld = a.ld[i];
        double *gA = a.A[i];
        const int tn = t + IRR_S_PF * stride;  // prefetch distance in items of this warp
        if (tn < count) {
            const int i2 = list[tn];
            const int m2 = a.m[i2], n2 = a.n[i2], ld2 = a.ld[i2];
            const char *p2 = reinterpret_cast<const char *>(a.A[i2]);
            const long bytes = ((long)(n2 - 1) * ld2 + m2) * 8;
            for (long o = (long)lane * 128; o < bytes; o += 32 * 128)
                asm volatile("prefetch.global.L2 [%0];" ::"l"(p2 + o));
        }
        lu_warp<NC>(gA, m, n, ld, a.ipiv[i], a.info + i, sm, lane);
    }
}

template <int NC>
static void launch_class(const GetrfArgs &a, const int *counters, const int *bins, cudaStream_t s) {
    const size_t smem = (size_t)S_WARPS * sizeof(SmallWarpSmem<NC>);
    smem_optin(lu_small_kernel<NC>, smem);
    int grid = num_sms() * SmallCfg<NC>::ctas;
    int need = (a.batch + S_WARPS - 1) / S_WARPS;
    if (grid > need) grid = need;
    if (grid < 1) grid = 1;
    KScope k(K_LU_SMALL, s);
    lu_small_kernel<NC><<<grid, 32 * S_WARPS, smem, s>>>(a, counters, bins);
}

// widest class first: it has the most work per matrix, the narrow kernels
// fill in behind it
void launch_lu_small(const GetrfArgs &a, const int *counters, const int *bins, cudaStream_t s,
                     const SmallStreams *ss) {
    const bool grouped = tuning().tier_s >= 2;
    const bool wide = a.max_n > 16 || a.max_m > 16 || !grouped;
    // the narrow classes on a second stream when the wide ones run too: each
    // class is a persistent grid, the second stream's CTAs take the SMs the
    // wide kernels' tails release
    cudaStream_t s2 = s;
    if (ss && wide && a.max_n > 0 && ss->s2 && cudaEventRecord(ss->fork, s) == cudaSuccess &&
        cudaStreamWaitEvent(ss->s2, ss->fork, 0) == cudaSuccess)
        s2 = ss->s2;
    if (wide) {
        launch_class<32>(a, counters, bins, s);
        if (grouped && a.max_n > 16) launch_class<24>(a, counters, bins, s);
    }
    if (a.max_n > 0) {
        if (a.max_m > 16 || !grouped) {
            launch_class<16>(a, counters, bins, s2);
            launch_class<8>(a, counters, bins, s2);
        }
        if (grouped) {
            if (a.max_m > 8 || a.max_n > 8) launch_group<16>(a, counters, bins, BIN_S16G, s2);
            launch_group<8>(a, counters, bins, BIN_S8G, s2);
        }
    }
    if (s2 != s) {
        cudaEventRecord(ss->join, s2);
        cudaStreamWaitEvent(s, ss->join, 0);
    }
}

}  // namespace irr

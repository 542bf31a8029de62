// gemm_core.cuh -- variable-size FP64 GEMM core with a device-side tile
// schedule (irrGEMM, §IV-C).
//
// Each problem slot b of a batch describes one (sub)matrix product after DCWI
// (P:L169).  A one-CTA scan kernel turns the per-slot tile counts into prefix
// offsets on the device; the persistent GEMM kernel then gives every CTA a
// contiguous range of the global tile index space (one binary search per CTA
// per launch), so there is neither a host loop over matrices nor a grid sized
// for the largest matrix with most CTAs idle.
//
// FP64 on sm_100a: tcgen05 has no f64 kind (SURVEY §7 hard part 4); the
// tensor path would be mma.sync DMMA whose peak equals the DFMA pipe.  This
// core uses DFMA with a 4x4 register tile per thread (64x64 CTA tile, K chunk
// 16, double-buffered shared memory).
#pragma once
#include "irr_internal.cuh"

namespace irr {

constexpr int GBM = 64, GBN = 64, GBK = 16, G_NT = 256;

struct GemmDesc {
    const double *A; long lda; int ta;
    const double *B; long ldb; int tb;
    double *C; long ldc;
    int m, n, k;
    double alpha, beta;
};

struct GemmSmem {
    double As[2][GBK][GBM + 1];
    double Bs[2][GBK][GBN + 1];
};

__device__ __forceinline__ void gemm_load_chunk(const GemmDesc &d, int r0, int c0, int k0, double (*As)[GBM + 1],
                                                double (*Bs)[GBN + 1], double ra[4], double rb[4]) {
    const int tid = threadIdx.x;
#pragma unroll
    for (int q = 0; q < 4; ++q) {
        const int e = tid + G_NT * q;
        int r, kk;
        if (!d.ta) { r = e & 63; kk = e >> 6; } else { kk = e & 15; r = e >> 4; }
        const int gr = r0 + r, gk = k0 + kk;
        double v = 0.0;
        if (gr < d.m && gk < d.k) v = d.ta ? d.A[gk + (size_t)gr * d.lda] : d.A[gr + (size_t)gk * d.lda];
        ra[q] = v;
    }
#pragma unroll
    for (int q = 0; q < 4; ++q) {
        const int e = tid + G_NT * q;
        int c, kk;
        if (!d.tb) { kk = e & 15; c = e >> 4; } else { c = e & 63; kk = e >> 6; }
        const int gc = c0 + c, gk = k0 + kk;
        double v = 0.0;
        if (gc < d.n && gk < d.k) v = d.tb ? d.B[gc + (size_t)gk * d.ldb] : d.B[gk + (size_t)gc * d.ldb];
        rb[q] = v;
    }
    (void)As; (void)Bs;
}

__device__ __forceinline__ void gemm_store_chunk(const GemmDesc &d, double (*As)[GBM + 1], double (*Bs)[GBN + 1],
                                                 const double ra[4], const double rb[4]) {
    const int tid = threadIdx.x;
#pragma unroll
    for (int q = 0; q < 4; ++q) {
        const int e = tid + G_NT * q;
        int r, kk;
        if (!d.ta) { r = e & 63; kk = e >> 6; } else { kk = e & 15; r = e >> 4; }
        As[kk][r] = ra[q];
    }
#pragma unroll
    for (int q = 0; q < 4; ++q) {
        const int e = tid + G_NT * q;
        int c, kk;
        if (!d.tb) { kk = e & 15; c = e >> 4; } else { c = e & 63; kk = e >> 6; }
        Bs[kk][c] = rb[q];
    }
}

// One 64x64 output tile at (r0, c0) of problem d:  C <- alpha op(A) op(B) + beta C
// (beta == 0: C is not read).  All G_NT threads participate.
__device__ __forceinline__ void gemm_tile(const GemmDesc &d, int r0, int c0, GemmSmem &sm) {
    const int tid = threadIdx.x, tx = tid & 15, ty = tid >> 4;
    double acc[4][4];
#pragma unroll
    for (int q = 0; q < 4; ++q)
#pragma unroll
        for (int p = 0; p < 4; ++p) acc[q][p] = 0.0;
    double ra[4], rb[4];
    int buf = 0;
    if (d.k > 0) {
        gemm_load_chunk(d, r0, c0, 0, sm.As[0], sm.Bs[0], ra, rb);
        gemm_store_chunk(d, sm.As[0], sm.Bs[0], ra, rb);
    }
    __syncthreads();
    for (int k0 = 0; k0 < d.k; k0 += GBK) {
        const bool has_next = k0 + GBK < d.k;
        if (has_next) gemm_load_chunk(d, r0, c0, k0 + GBK, sm.As[buf ^ 1], sm.Bs[buf ^ 1], ra, rb);
#pragma unroll
        for (int kk = 0; kk < GBK; ++kk) {
            double a[4], b[4];
#pragma unroll
            for (int q = 0; q < 4; ++q) a[q] = sm.As[buf][kk][tx + 16 * q];
#pragma unroll
            for (int p = 0; p < 4; ++p) b[p] = sm.Bs[buf][kk][ty + 16 * p];
#pragma unroll
            for (int q = 0; q < 4; ++q)
#pragma unroll
                for (int p = 0; p < 4; ++p) acc[q][p] = fma(a[q], b[p], acc[q][p]);
        }
        if (has_next) gemm_store_chunk(d, sm.As[buf ^ 1], sm.Bs[buf ^ 1], ra, rb);
        __syncthreads();
        buf ^= 1;
    }
#pragma unroll
    for (int p = 0; p < 4; ++p) {
        const int c = c0 + ty + 16 * p;
        if (c >= d.n) continue;
#pragma unroll
        for (int q = 0; q < 4; ++q) {
            const int r = r0 + tx + 16 * q;
            if (r >= d.m) continue;
            double *cp = d.C + r + (size_t)c * d.ldc;
            *cp = (d.beta == 0.0) ? d.alpha * acc[q][p] : d.alpha * acc[q][p] + d.beta * *cp;
        }
    }
}

__device__ __forceinline__ int gemm_tiles_of(const GemmDesc &d) {
    if (d.m <= 0 || d.n <= 0) return 0;
    return ((d.m + GBM - 1) / GBM) * ((d.n + GBN - 1) / GBN);
}

// count: number of problem slots, from *count_ptr when count < 0.
template <class Prob>
__global__ void __launch_bounds__(1024) gemm_scan_kernel(Prob P, int count, const int *count_ptr, int *tile_off) {
    __shared__ int warp_sums[32];
    __shared__ int carry_s;
    if (count < 0) count = *count_ptr;
    const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
    if (tid == 0) carry_s = 0;
    __syncthreads();
    for (int base = 0; base < count; base += 1024) {
        const int b = base + tid;
        int v = 0;
        if (b < count) {
            GemmDesc d;
            if (P.get(b, d)) v = gemm_tiles_of(d);
        }
        int x = v;
#pragma unroll
        for (int o = 1; o < 32; o <<= 1) {
            int y = __shfl_up_sync(FULL, x, o);
            if (lane >= o) x += y;
        }
        if (lane == 31) warp_sums[warp] = x;
        __syncthreads();
        if (warp == 0) {
            int w = warp_sums[lane];
#pragma unroll
            for (int o = 1; o < 32; o <<= 1) {
                int y = __shfl_up_sync(FULL, w, o);
                if (lane >= o) w += y;
            }
            warp_sums[lane] = w;  // inclusive
        }
        __syncthreads();
        const int carry = carry_s;
        const int excl = carry + (warp ? warp_sums[warp - 1] : 0) + x - v;
        if (b < count) tile_off[b] = excl;
        __syncthreads();
        if (tid == 1023) carry_s = excl + v;
        __syncthreads();
    }
    if (tid == 0) tile_off[count] = carry_s;
}

template <class Prob>
__global__ void __launch_bounds__(G_NT) gemm_sched_kernel(Prob P, int count, const int *count_ptr,
                                                          const int *__restrict__ tile_off) {
    __shared__ GemmSmem sm;
    if (count < 0) count = *count_ptr;
    if (count <= 0) return;
    const int total = tile_off[count];
    const long long G = gridDim.x;
    const int t_begin = (int)((long long)blockIdx.x * total / G);
    const int t_end = (int)((long long)(blockIdx.x + 1) * total / G);
    if (t_begin >= t_end) return;
    // first slot b with tile_off[b] <= t_begin < tile_off[b+1]
    int lo = 0, hi = count - 1;
    while (lo < hi) {
        int mid = (lo + hi + 1) >> 1;
        if (tile_off[mid] <= t_begin) lo = mid; else hi = mid - 1;
    }
    int b = lo;
    GemmDesc d;
    P.get(b, d);
    int b_end = tile_off[b + 1];
    for (int t = t_begin; t < t_end; ++t) {
        while (t >= b_end) {
            ++b;
            P.get(b, d);
            b_end = tile_off[b + 1];
        }
        const int local = t - tile_off[b];
        const int ntm = (d.m + GBM - 1) / GBM;
        const int tm = local % ntm, tn = local / ntm;
        gemm_tile(d, tm * GBM, tn * GBN, sm);
        __syncthreads();
    }
}

// DCWI-grid fallback (no workspace): virtual tiles over the required dims,
// empty ones exit immediately ("If no workload is detected, the
// corresponding GPU threads perform no work at all").
template <class Prob>
__global__ void __launch_bounds__(G_NT) gemm_grid_kernel(Prob P, int count, int tiles_m, int tiles_n) {
    __shared__ GemmSmem sm;
    const long long per = (long long)tiles_m * tiles_n;
    const long long total = per * count;
    for (long long w = blockIdx.x; w < total; w += gridDim.x) {
        const int b = (int)(w / per);
        const int local = (int)(w - (long long)b * per);
        GemmDesc d;
        if (!P.get(b, d)) continue;
        const int tm = local % tiles_m, tn = local / tiles_m;
        if (tm * GBM >= d.m || tn * GBN >= d.n) continue;
        gemm_tile(d, tm * GBM, tn * GBN, sm);
        __syncthreads();
    }
}

}  // namespace irr

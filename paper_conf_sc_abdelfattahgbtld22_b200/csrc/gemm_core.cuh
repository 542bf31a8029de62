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
// tensor path would be mma.sync DMMA whose nominal peak equals the DFMA pipe.
// This core uses DFMA: 64x64 CTA tile, 128 threads, 8x4 register tile per
// thread (12 shared-memory wavefronts per 32 DFMA, below the 1:2 ratio the
// SM sustains), operands staged by cp.async in K chunks of 16 with double
// buffering, the C tile staged asynchronously, and the next tile's first
// chunk prefetched while the current tile computes.
#pragma once
#include "irr_internal.cuh"

namespace irr {

constexpr int GBM = 64, GBN = 64, GBK = 16, G_NT = 128;
constexpr int GPAD = GBM + 2;  // even: 16-byte row pairs of the A stage stay aligned; 2-way (not 4-way) fragment conflicts

struct GemmDesc {
    const double *A; long lda; int ta;
    const double *B; long ldb; int tb;
    double *C; long ldc;
    int m, n, k;
    double alpha, beta;
};

constexpr int CPAD = GBM + 2;  // even: 16-byte row pairs of the C stage stay aligned (cp.async16, LDS.128)

struct GemmSmem {
    double As[2][GBK][GPAD];
    double Bs[2][GBK][GPAD];
    double Cs[GBN][CPAD];
};
constexpr size_t GEMM_SMEM = sizeof(GemmSmem);

// Issue the cp.async copies of K chunk [k0, k0+16) of tile (r0, c0) into buffer
// `buf` (out-of-range elements are zero-filled with plain stores).
template <bool BRES = false, bool APAIR = true>
__device__ __forceinline__ void gemm_issue_chunk(const GemmDesc &d, int r0, int c0, int k0, GemmSmem &sm, int buf) {
    const int tid = threadIdx.x;
    if (APAIR && !d.ta) {
        // op(A) = A column-major: row pairs (2p, 2p+1) of column kk, one
        // 16-byte copy where the pair is aligned in global memory, else two
#pragma unroll
        for (int q = 0; q < (GBM * GBK) / (2 * G_NT); ++q) {
            const int e = tid + G_NT * q;
            const int r = 2 * (e & 31), kk = e >> 5;
            const int gr = r0 + r, gk = k0 + kk;
            double *dst = &sm.As[buf][kk][r];
            const double *src = d.A + gr + (size_t)gk * d.lda;
            const bool okk = gk < d.k;
            if (okk && gr + 1 < d.m && ((reinterpret_cast<uintptr_t>(src) & 15) == 0)) {
                cp_async16(dst, src);
            } else {
                if (okk && gr < d.m) cp_async8(dst, src); else dst[0] = 0.0;
                if (okk && gr + 1 < d.m) cp_async8(dst + 1, src + 1); else dst[1] = 0.0;
            }
        }
    } else {
#pragma unroll
    for (int q = 0; q < (GBM * GBK) / G_NT; ++q) {
        const int e = tid + G_NT * q;
        int r, kk;
        if (!d.ta) { r = e & 63; kk = e >> 6; } else { kk = e & 15; r = e >> 4; }
        const int gr = r0 + r, gk = k0 + kk;
        double *dst = &sm.As[buf][kk][r];
        if (gr < d.m && gk < d.k) {
            cp_async8(dst, d.ta ? d.A + gk + (size_t)gr * d.lda : d.A + gr + (size_t)gk * d.lda);
        } else {
            *dst = 0.0;
        }
    }
    }
    if (BRES) return;  // B already resident in sm.Bs (the caller staged all K rows)
#pragma unroll
    for (int q = 0; q < (GBN * GBK) / G_NT; ++q) {
        const int e = tid + G_NT * q;
        int c, kk;
        if (!d.tb) { kk = e & 15; c = e >> 4; } else { c = e & 63; kk = e >> 6; }
        const int gc = c0 + c, gk = k0 + kk;
        double *dst = &sm.Bs[buf][kk][c];
        if (gc < d.n && gk < d.k) {
            cp_async8(dst, d.tb ? d.B + gc + (size_t)gk * d.ldb : d.B + gk + (size_t)gc * d.ldb);
        } else {
            *dst = 0.0;
        }
    }
}

__device__ __forceinline__ void gemm_issue_c(const GemmDesc &d, int r0, int c0, GemmSmem &sm) {
    if (d.beta == 0.0) return;
    const int tid = threadIdx.x;
    const int mr = imin(GBM, d.m - r0), nc = imin(GBN, d.n - c0);
    // row pair (2p, 2p+1) per thread: one 16-byte copy where the column's
    // pair is 16-byte aligned in global memory (parity of r0 + c ldc), else two
    const int p2 = 2 * (tid & 31);
    if (p2 >= mr) return;
    const bool two = p2 + 1 < mr;
    for (int c = tid >> 5; c < nc; c += G_NT / 32) {
        const double *src = d.C + r0 + p2 + (size_t)(c0 + c) * d.ldc;
        double *dst = &sm.Cs[c][p2];
        if (two && ((reinterpret_cast<uintptr_t>(src) & 15) == 0)) {
            cp_async16(dst, src);
        } else {
            cp_async8(dst, src);
            if (two) cp_async8(dst + 1, src + 1);
        }
    }
}

// ---- DFMA path: thread (tx, ty) owns rows tx + 8q (q < 8), cols ty + 16p (p < 4);
//      acc[q * 4 + p].  12 shared-memory wavefronts per 32 DFMA per warp.
__device__ __forceinline__ void gemm_compute_chunk_dfma(const GemmSmem &sm, int buf, double (&acc)[32],
                                                        int bbuf = -1) {
    if (bbuf < 0) bbuf = buf;
    const int tid = threadIdx.x, tx = tid & 7, ty = tid >> 3;
#pragma unroll
    for (int kk = 0; kk < GBK; ++kk) {
        double a[8], b[4];
#pragma unroll
        for (int q = 0; q < 8; ++q) a[q] = sm.As[buf][kk][tx + 8 * q];
#pragma unroll
        for (int p = 0; p < 4; ++p) b[p] = sm.Bs[bbuf][kk][ty + 16 * p];
#pragma unroll
        for (int q = 0; q < 8; ++q)
#pragma unroll
            for (int p = 0; p < 4; ++p) acc[q * 4 + p] = fma(a[q], b[p], acc[q * 4 + p]);
    }
}

// ---- DMMA path (FP64 tensor core, mma.sync m8n8k4 -> SASS DMMA.8x8x4):
//      warp w computes the 32x32 sub-tile (rows 32 (w&1), cols 32 (w>>1)) as
//      4 x 4 mma tiles; lane (g = lane>>2, t = lane&3) loads A(g, t) and B(t, g)
//      and the mma runs TRANSPOSED (C^T = B^T A^T: B's fragment as the row
//      operand), so acc[(mi * 4 + ni) * 2 + i] = C(8 mi + 2t + i, 8 ni + g):
//      two adjacent rows of one column, i.e. one 16-byte global access in the
//      column-major C.  One DMMA = 256 FMA; two 8-byte loads per lane per 16 DMMA.
__device__ __forceinline__ void dmma_8x8x4(double &c0, double &c1, double a, double b) {
    asm volatile("mma.sync.aligned.m8n8k4.row.col.f64.f64.f64.f64 {%0,%1}, {%2}, {%3}, {%0,%1};\n"
                 : "+d"(c0), "+d"(c1)
                 : "d"(a), "d"(b));
}

__device__ __forceinline__ void gemm_compute_chunk_dmma(const GemmSmem &sm, int buf, double (&acc)[32],
                                                        int bbuf = -1) {
    if (bbuf < 0) bbuf = buf;
    const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
    const int g = lane >> 2, t = lane & 3;
    const int rb = (warp & 1) * 32 + g, cb = (warp >> 1) * 32 + g;
#pragma unroll
    for (int ks = 0; ks < GBK; ks += 4) {
        double a[4], b[4];
#pragma unroll
        for (int mi = 0; mi < 4; ++mi) a[mi] = sm.As[buf][ks + t][rb + 8 * mi];
#pragma unroll
        for (int ni = 0; ni < 4; ++ni) b[ni] = sm.Bs[bbuf][ks + t][cb + 8 * ni];
#pragma unroll
        for (int mi = 0; mi < 4; ++mi)
#pragma unroll
            for (int ni = 0; ni < 4; ++ni)
                dmma_8x8x4(acc[(mi * 4 + ni) * 2], acc[(mi * 4 + ni) * 2 + 1], b[ni], a[mi]);
    }
}

// DMMA path without a shared-memory C stage: this lane's 32 C values go
// straight from global memory into registers, issued at the start of the tile
// and consumed by the epilogue (ncu, strip kernel on C3: the epilogue's wait
// on the staged C tile was the largest stall, 16%).  Measured SLOWER on B200
// (C3 strip 57.8 -> 60.4 ms, C2 6.44 -> 6.54 ms), so off by default (CREG_OK).
__device__ __forceinline__ void gemm_load_c_regs(const GemmDesc &d, int r0, int c0, double (&cr)[32]) {
    const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
    const int g = lane >> 2, t = lane & 3;
    const bool rd = d.beta != 0.0;
#pragma unroll
    for (int mi = 0; mi < 4; ++mi) {
#pragma unroll
        for (int ni = 0; ni < 4; ++ni) {
            const int c = c0 + (warp >> 1) * 32 + 8 * ni + g;
#pragma unroll
            for (int i = 0; i < 2; ++i) {
                const int r = r0 + (warp & 1) * 32 + 8 * mi + 2 * t + i;
                cr[(mi * 4 + ni) * 2 + i] = (rd && r < d.m && c < d.n) ? d.C[r + (size_t)c * d.ldc] : 0.0;
            }
        }
    }
}

__device__ __forceinline__ void gemm_epilogue_creg(const GemmDesc &d, int r0, int c0, const double (&acc)[32],
                                                   const double (&cr)[32]) {
    const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
    const int g = lane >> 2, t = lane & 3;
#pragma unroll
    for (int mi = 0; mi < 4; ++mi) {
#pragma unroll
        for (int ni = 0; ni < 4; ++ni) {
            const int c = c0 + (warp >> 1) * 32 + 8 * ni + g;
            if (c >= d.n) continue;
#pragma unroll
            for (int i = 0; i < 2; ++i) {
                const int r = r0 + (warp & 1) * 32 + 8 * mi + 2 * t + i;
                if (r >= d.m) continue;
                const int q = (mi * 4 + ni) * 2 + i;
                double v = d.alpha * acc[q];
                if (d.beta != 0.0) v = fma(d.beta, cr[q], v);
                d.C[r + (size_t)c * d.ldc] = v;
            }
        }
    }
}

template <bool DMMA>
__device__ __forceinline__ void gemm_epilogue(const GemmDesc &d, int r0, int c0, const GemmSmem &sm,
                                              const double (&acc)[32]) {
    const int tid = threadIdx.x;
    if (!DMMA) {
        const int tx = tid & 7, ty = tid >> 3;
#pragma unroll
        for (int q = 0; q < 8; ++q) {
            const int rl = tx + 8 * q, r = r0 + rl;
            if (r >= d.m) continue;
#pragma unroll
            for (int p = 0; p < 4; ++p) {
                const int cl = ty + 16 * p, c = c0 + cl;
                if (c >= d.n) continue;
                double v = d.alpha * acc[q * 4 + p];
                if (d.beta != 0.0) v += d.beta * sm.Cs[cl][rl];
                d.C[r + (size_t)c * d.ldc] = v;
            }
        }
    } else {
        // lane holds C(rl, cl) and C(rl + 1, cl): one 16-byte store where the
        // pair is aligned and both rows exist, else two 8-byte stores
        const int lane = tid & 31, warp = tid >> 5;
        const int g = lane >> 2, t = lane & 3;
        const bool rdc = d.beta != 0.0;
#pragma unroll
        for (int ni = 0; ni < 4; ++ni) {
            const int cl = (warp >> 1) * 32 + 8 * ni + g, c = c0 + cl;
            if (c >= d.n) continue;
#pragma unroll
            for (int mi = 0; mi < 4; ++mi) {
                const int rl = (warp & 1) * 32 + 8 * mi + 2 * t, r = r0 + rl;
                if (r >= d.m) continue;
                const int q = (mi * 4 + ni) * 2;
                double v0 = d.alpha * acc[q], v1 = d.alpha * acc[q + 1];
                if (rdc) {  // rl even and CPAD even: the pair is one 16-byte shared load
                    const double2 cv = *reinterpret_cast<const double2 *>(&sm.Cs[cl][rl]);
                    v0 = fma(d.beta, cv.x, v0);
                    v1 = fma(d.beta, cv.y, v1);
                }
                double *dst = d.C + r + (size_t)c * d.ldc;
                if (r + 1 < d.m && ((reinterpret_cast<uintptr_t>(dst) & 15) == 0)) {
                    *reinterpret_cast<double2 *>(dst) = make_double2(v0, v1);
                } else {
                    dst[0] = v0;
                    if (r + 1 < d.m) dst[1] = v1;
                }
            }
        }
    }
}

// A stream of tiles processed by one CTA with the software pipeline described
// above.  `next(d, r0, c0)` returns false when the CTA has no more tiles.
// DMMA selects the FP64 tensor-core path, else DFMA.
// BRES: op(B) (k <= 2 GBK rows) is resident in sm.Bs for every tile of the
// stream -- chunk c reads Bs[c] -- and is never loaded (the strip kernel's
// U12, solved in place there).
// APAIR: 16-byte row-pair copies of op(A) (off where the extra registers spill).
template <bool DMMA, class Next, bool CREG_OK = false, bool BRES = false, bool APAIR = true>
__device__ __forceinline__ void gemm_tile_stream(Next next, GemmSmem &sm) {
    GemmDesc d, dn;
    int r0, c0, rn, cn;
    if (!next(d, r0, c0)) return;
    int buf = 0;
    if (d.k > 0) gemm_issue_chunk<BRES, APAIR>(d, r0, c0, 0, sm, buf);
    cp_async_commit();
    bool have = true;
    constexpr bool CREG = DMMA && CREG_OK;  // C in registers (the commit below is then an empty group)
    while (have) {
        double cr[32];
        if (CREG) gemm_load_c_regs(d, r0, c0, cr);
        else gemm_issue_c(d, r0, c0, sm);
        cp_async_commit();
        double acc[32];
#pragma unroll
        for (int q = 0; q < 32; ++q) acc[q] = 0.0;
        const int nchunks = (d.k + GBK - 1) / GBK;
        bool has_next_tile = false;
        for (int c = 0; c < (nchunks > 0 ? nchunks : 1); ++c) {
            if (c + 1 < nchunks) {
                gemm_issue_chunk<BRES, APAIR>(d, r0, c0, (c + 1) * GBK, sm, buf ^ 1);
            } else {
                has_next_tile = next(dn, rn, cn);
                if (has_next_tile && dn.k > 0) gemm_issue_chunk<BRES, APAIR>(dn, rn, cn, 0, sm, buf ^ 1);
            }
            cp_async_commit();
            if (c == 0) cp_async_wait<2>(); else cp_async_wait<1>();
            __syncthreads();
            if (nchunks > 0) {
                if (DMMA) gemm_compute_chunk_dmma(sm, buf, acc, BRES ? c : buf);
                else gemm_compute_chunk_dfma(sm, buf, acc, BRES ? c : buf);
            }
            __syncthreads();
            buf ^= 1;
        }
        if (CREG) {
            gemm_epilogue_creg(d, r0, c0, acc, cr);
        } else {
            cp_async_wait<1>();
            __syncthreads();
            gemm_epilogue<DMMA>(d, r0, c0, sm, acc);
            __syncthreads();
        }
        have = has_next_tile;
        if (have) { d = dn; r0 = rn; c0 = cn; }
    }
    cp_async_wait<0>();
}

__device__ __forceinline__ int gemm_tiles_of(const GemmDesc &d) {
    if (d.m <= 0 || d.n <= 0) return 0;
    return ((d.m + GBM - 1) / GBM) * ((d.n + GBN - 1) / GBN);
}

// Schedule weight of one tile: its K chunks in units of 128 plus one for the C
// tile (tiles of a batch differ in K by 100x in a multifrontal batch; equal
// tile counts per CTA left the CTAs holding the big fronts 1.75x over).
__device__ __forceinline__ int gemm_tile_weight(const GemmDesc &d) { return 1 + (d.k > 0 ? (d.k + 127) / 128 : 0); }

// count: number of problem slots, from *count_ptr when count < 0.
// tile_off[b] = weighted work before slot b (gemm_tile_weight units).
// C fragments in registers for the DMMA epilogue (gemm_load_c_regs) where the
// problem's descriptor code leaves the register room (the DCWI descriptor
// spills with it); specialised next to the problem types that opt in.
template <class Prob>
struct gemm_creg_ok { static constexpr bool value = false; };

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
            if (P.get(b, d)) v = gemm_tiles_of(d) * gemm_tile_weight(d);
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

template <class Prob, bool DMMA>
__global__ void __launch_bounds__(G_NT, 3) gemm_sched_kernel(Prob P, int count, const int *count_ptr,
                                                          const int *__restrict__ tile_off) {
    extern __shared__ __align__(16) unsigned char g_smem[];
    GemmSmem &sm = *reinterpret_cast<GemmSmem *>(g_smem);
    if (count < 0) count = *count_ptr;
    if (count <= 0) return;
    const int total = tile_off[count];
    const long long G = gridDim.x;
    // this CTA owns the tiles whose weighted start lies in [u_begin, u_end)
    const int u_begin = (int)((long long)blockIdx.x * total / G);
    const int u_end = (int)((long long)(blockIdx.x + 1) * total / G);
    if (u_begin >= u_end) return;
    int lo = 0, hi = count - 1;  // last slot b with tile_off[b] <= u_begin
    while (lo < hi) {
        int mid = (lo + hi + 1) >> 1;
        if (tile_off[mid] <= u_begin) lo = mid; else hi = mid - 1;
    }
    int b = lo;
    GemmDesc cur;
    P.get(b, cur);
    int w = gemm_tile_weight(cur), off_b = tile_off[b];
    int nt_b = (tile_off[b + 1] - off_b) / w;
    int local = u_begin > off_b ? (u_begin - off_b + w - 1) / w : 0;
    auto next = [&](GemmDesc &d, int &r0, int &c0) -> bool {
        while (local >= nt_b) {
            if (++b >= count) return false;
            off_b = tile_off[b];
            if (off_b >= u_end) return false;
            P.get(b, cur);
            w = gemm_tile_weight(cur);
            nt_b = (tile_off[b + 1] - off_b) / w;
            local = 0;
        }
        if (off_b + local * w >= u_end) return false;
        const int ntm = (cur.m + GBM - 1) / GBM;
        r0 = (local % ntm) * GBM;
        c0 = (local / ntm) * GBN;
        d = cur;
        ++local;
        return true;
    };
    gemm_tile_stream<DMMA, decltype(next), gemm_creg_ok<Prob>::value>(next, sm);
}

// DCWI-grid fallback (no workspace): virtual tiles over the required dims,
// empty ones are skipped ("If no workload is detected, the
// corresponding GPU threads perform no work at all").
template <class Prob, bool DMMA>
__global__ void __launch_bounds__(G_NT, 3) gemm_grid_kernel(Prob P, int count, int tiles_m, int tiles_n) {
    extern __shared__ __align__(16) unsigned char g_smem[];
    GemmSmem &sm = *reinterpret_cast<GemmSmem *>(g_smem);
    const long long per = (long long)tiles_m * tiles_n;
    const long long total = per * count;
    long long w = blockIdx.x;
    auto next = [&](GemmDesc &d, int &r0, int &c0) -> bool {
        for (; w < total; w += gridDim.x) {
            const int b = (int)(w / per);
            const int local = (int)(w - (long long)b * per);
            if (!P.get(b, d)) continue;
            const int tm = local % tiles_m, tn = local / tiles_m;
            if (tm * GBM >= d.m || tn * GBN >= d.n) continue;
            r0 = tm * GBM;
            c0 = tn * GBN;
            w += gridDim.x;
            return true;
        }
        return false;
    };
    gemm_tile_stream<DMMA>(next, sm);
}

// opt-in to > 48 KB dynamic shared memory once per kernel instantiation
template <class K>
inline void gemm_smem_optin(K kernel) {
    smem_optin(kernel, GEMM_SMEM);
}

}  // namespace irr

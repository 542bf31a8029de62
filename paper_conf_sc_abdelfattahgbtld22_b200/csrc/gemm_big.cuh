// gemm_big.cuh -- the large-tile FP64 tensor-core GEMM core of irrGEMM
// (§IV-C; SURVEY §8(a) a5.3 and the TRSM recursion of a5.2).
//
// The partial front factorization spends 58% of its flops in F22 -= F21 F12
// with K = n1 up to ~2000 and another 35% in the off-diagonal GEMMs of the
// recursive TRSM ("runtime most impacted by the GEMM performance on
// the largest nodes").  For those long-K products the 64 x 64 core
// (gemm_core.cuh) is bound by its operand traffic; this core is sized for
// the DMMA pipe instead:
//   * 128 x 128 CTA tile, 256 threads = 8 warps in a 2 x 4 grid, each warp a
//     64 x 32 tile of 8 x 4 mma.sync.m8n8k4.f64 (SASS DMMA.884) accumulators
//     (64 doubles per lane), so one k-step is 12 fragment loads per 32 DMMA;
//   * K chunks of 16 staged by cp.async in a 4-deep ring (one barrier per
//     chunk), shared layouts chosen per transpose so every fragment load is
//     bank-conflict free: k-major [k][m] with ld 132 when the operand is
//     contiguous along m (n), m-major [m][k] with ld 20 when contiguous along k;
//   * 1 CTA per SM (8 warps saturate DMMA: profiles/r01/microbench.txt),
//     persistent over a device tile schedule weighted by K.
// Epilogue reads / writes C straight from registers (each warp store covers
// 64-byte column segments).
#pragma once
#include "gemm_core.cuh"

namespace irr {

#ifndef XGEMM_ST
#define XGEMM_ST 4      // cp.async ring depth (K chunks in flight)
#endif
#ifndef XGEMM_MINB
#define XGEMM_MINB 1    // resident CTAs per SM
#endif
#ifndef XGEMM_BK
#define XGEMM_BK 16     // K chunk per ring stage
#endif
constexpr int XBM = 128, XBN = 128, XBK = XGEMM_BK, X_NT = 256, XST = XGEMM_ST;
constexpr int XLD_KM = 132;  // [k][m] layout: XBK rows of XBM (+4)
constexpr int XLD_MK = XBK + 4;   // [m][k] layout: XBM rows of XBK (+4)
constexpr int XSTAGE = (XBK * XLD_KM > XBM * XLD_MK) ? XBK * XLD_KM : XBM * XLD_MK;  // doubles per operand stage

struct BigSmem {
    double A[XST][XSTAGE];
    double B[XST][XSTAGE];
};
constexpr size_t BIG_SMEM = sizeof(BigSmem);

// cp.async with zero fill: src_bytes = 0 writes zeros and reads nothing
__device__ __forceinline__ void cp_async8_zf(void *smem, const void *gmem, bool valid) {
    unsigned s = (unsigned)__cvta_generic_to_shared(smem);
    const int n = valid ? 8 : 0;
    asm volatile("cp.async.ca.shared.global [%0], [%1], 8, %2;\n" ::"r"(s), "l"(gmem), "r"(n) : "memory");
}

// 16-byte copy of elements (i, i+1) along the operand's contiguous dimension
// when both exist and the source pair is aligned, else 8-byte copies / zeros
// (`base`: an in-bounds address for the zero-filling copies, never read)
__device__ __forceinline__ void x_pair(double *dst, const double *src, bool ok0, bool ok1, const double *base) {
    if (ok0 && ok1 && ((reinterpret_cast<uintptr_t>(src) & 15) == 0)) {
        cp_async16(dst, src);
    } else {
        cp_async8_zf(dst, ok0 ? src : base, ok0);
        cp_async8_zf(dst + 1, ok1 ? src + 1 : base, ok1);
    }
}

// Stage chunk [k0, k0+16) of the (r0, c0) tile.  op(A) is m x k, op(B) k x n.
// Element pairs along each operand's contiguous dimension (m for A, k for
// A^T, k for B, n for B^T): both shared layouts keep such pairs 16-byte
// aligned (even leading dimensions 132 / 20).
template <int TA, int TB, int NT = X_NT>
__device__ __forceinline__ void xgemm_issue(const GemmDesc &d, int r0, int c0, int k0, BigSmem &sm, int st,
                                            int tid = -1, bool skip_a = false) {
    if (tid < 0) tid = threadIdx.x;
    double *As = sm.A[st];
    double *Bs = sm.B[st];
#pragma unroll
    for (int q = 0; q < (XBM * XBK) / (2 * NT); ++q) {
        if (skip_a) break;
        const int e = tid + NT * q;
        if (!TA) {  // A(m, k) at A + m + k lda: pairs along m
            const int m = 2 * (e & (XBM / 2 - 1)), kk = e / (XBM / 2);
            const int gm = r0 + m, gk = k0 + kk;
            const bool okk = gk < d.k;
            x_pair(&As[kk * XLD_KM + m], d.A + gm + (size_t)(okk ? gk : 0) * d.lda, okk && gm < d.m,
                   okk && gm + 1 < d.m, d.A);
        } else {    // A(k, m) at A + k + m lda: pairs along k
            const int kk = 2 * (e & (XBK / 2 - 1)), m = e / (XBK / 2);
            const int gm = r0 + m, gk = k0 + kk;
            const bool okm = gm < d.m;
            x_pair(&As[m * XLD_MK + kk], d.A + gk + (size_t)(okm ? gm : 0) * d.lda, okm && gk < d.k,
                   okm && gk + 1 < d.k, d.A);
        }
    }
#pragma unroll
    for (int q = 0; q < (XBN * XBK) / (2 * NT); ++q) {
        const int e = tid + NT * q;
        if (!TB) {  // B(k, n) at B + k + n ldb: pairs along k
            const int kk = 2 * (e & (XBK / 2 - 1)), n = e / (XBK / 2);
            const int gn = c0 + n, gk = k0 + kk;
            const bool okn = gn < d.n;
            x_pair(&Bs[n * XLD_MK + kk], d.B + gk + (size_t)(okn ? gn : 0) * d.ldb, okn && gk < d.k,
                   okn && gk + 1 < d.k, d.B);
        } else {    // B(n, k) at B + n + k ldb: pairs along n
            const int n = 2 * (e & (XBN / 2 - 1)), kk = e / (XBN / 2);
            const int gn = c0 + n, gk = k0 + kk;
            const bool okk = gk < d.k;
            x_pair(&Bs[kk * XLD_KM + n], d.B + gn + (size_t)(okk ? gk : 0) * d.ldb, okk && gn < d.n,
                   okk && gn + 1 < d.n, d.B);
        }
    }
}

// NWG warps: 8 -> a 2 x 4 warp grid of 64 x 32 warp tiles (MI = 8 mma rows),
// 16 -> 4 x 4 warps of 32 x 32 (MI = 4): more warps to hide the DMMA /
// fragment-load latencies at half the accumulators per thread.
template <int NWG>
struct XWarp {
    static constexpr int MI = NWG == 16 ? 4 : 8;
    static constexpr int WGM = NWG == 16 ? 4 : 2;   // warps along m
    static constexpr int ACC = MI * 4 * 2;
};

template <int TA, int TB, int NWG = 8>
__device__ __forceinline__ void xgemm_compute(const BigSmem &sm, int st, double (&acc)[XWarp<NWG>::ACC],
                                              int aoff = 0) {
    constexpr int MI = XWarp<NWG>::MI, WGM = XWarp<NWG>::WGM;
    const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
    const int g = lane >> 2, t = lane & 3;
    const int wm = (warp % WGM) * (8 * MI), wn = (warp / WGM) * 32;
    const double *As = sm.A[st];
    const double *Bs = sm.B[st];
#pragma unroll
    for (int ks = 0; ks < XBK; ks += 4) {
        double a[MI], b[4];
#pragma unroll
        for (int mi = 0; mi < MI; ++mi) {
            const int m = wm + 8 * mi + g, k = ks + t;
            a[mi] = TA ? As[m * XLD_MK + k] : As[k * XLD_KM + m + aoff];
        }
#pragma unroll
        for (int ni = 0; ni < 4; ++ni) {
            const int n = wn + 8 * ni + g, k = ks + t;
            b[ni] = TB ? Bs[k * XLD_KM + n] : Bs[n * XLD_MK + k];
        }
#pragma unroll
        for (int mi = 0; mi < MI; ++mi)
#pragma unroll
            for (int ni = 0; ni < 4; ++ni)
                dmma_8x8x4(acc[(mi * 4 + ni) * 2], acc[(mi * 4 + ni) * 2 + 1], a[mi], b[ni]);
    }
}

template <int NWG = 8>
__device__ __forceinline__ void xgemm_epilogue(const GemmDesc &d, int r0, int c0,
                                               const double (&acc)[XWarp<NWG>::ACC]) {
    constexpr int MI = XWarp<NWG>::MI, WGM = XWarp<NWG>::WGM;
    const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
    const int g = lane >> 2, t = lane & 3;
    const int wm = (warp % WGM) * (8 * MI), wn = (warp / WGM) * 32;
    const bool rd = d.beta != 0.0;
    // two 8-row groups per round: 16 loads of C in flight before the stores
    // (the compiler cannot move later loads above the stores: same array)
#pragma unroll
    for (int m2 = 0; m2 < MI; m2 += 2) {
        double cv[2][8];
        if (rd) {
#pragma unroll
            for (int h = 0; h < 2; ++h) {
                const int r = r0 + wm + 8 * (m2 + h) + g;
#pragma unroll
                for (int ni = 0; ni < 4; ++ni)
#pragma unroll
                    for (int i = 0; i < 2; ++i) {
                        const int c = c0 + wn + 8 * ni + 2 * t + i;
                        cv[h][ni * 2 + i] = (r < d.m && c < d.n) ? d.C[r + (size_t)c * d.ldc] : 0.0;
                    }
            }
        }
#pragma unroll
        for (int h = 0; h < 2; ++h) {
            const int mi = m2 + h;
            const int r = r0 + wm + 8 * mi + g;
            if (r >= d.m) continue;
#pragma unroll
            for (int ni = 0; ni < 4; ++ni)
#pragma unroll
                for (int i = 0; i < 2; ++i) {
                    const int c = c0 + wn + 8 * ni + 2 * t + i;
                    if (c >= d.n) continue;
                    double v = d.alpha * acc[(mi * 4 + ni) * 2 + i];
                    if (rd) v = fma(d.beta, cv[h][ni * 2 + i], v);
                    d.C[r + (size_t)c * d.ldc] = v;
                }
        }
    }
}

// C tile -> L2 at the start of the tile (one 128-byte line = 16 rows of a
// column per prefetch, 4 per thread), so the epilogue's loads hit L2 instead
// of HBM; the DMMA pipe idles during the epilogue of this 1-CTA/SM core.
template <int NT = X_NT>
__device__ __forceinline__ void xgemm_prefetch_c(const GemmDesc &d, int r0, int c0) {
    if (d.beta == 0.0) return;
    constexpr int GR = XBM / (NT / 128);   // rows per thread group
    const int tid = threadIdx.x;
    const int c = c0 + (tid & 127);
    if (c >= d.n) return;
#pragma unroll
    for (int q = 0; q < GR / 16; ++q) {
        const int r = r0 + (tid >> 7) * GR + 16 * q;
        if (r < d.m) asm volatile("prefetch.global.L2 [%0];" ::"l"(d.C + r + (size_t)c * d.ldc));
    }
}

// Ring prologue of a tile: its C tile towards L2 and its first XST-1 K chunks.
template <int TA, int TB, int NT>
__device__ __forceinline__ void xgemm_prologue(const GemmDesc &d, int r0, int c0, BigSmem &sm) {
    const int nk = (d.k + XBK - 1) / XBK;
    xgemm_prefetch_c<NT>(d, r0, c0);
#pragma unroll
    for (int s = 0; s < XST - 1; ++s) {
        if (s < nk) xgemm_issue<TA, TB, NT>(d, r0, c0, s * XBK, sm, s);
        cp_async_commit();
    }
}

// The K loop of a tile whose prologue has been issued.  Ends with the ring
// free (every chunk consumed, barrier passed), the product in acc.
template <int TA, int TB, int NWG = 8>
__device__ __forceinline__ void xgemm_main(const GemmDesc &d, int r0, int c0, BigSmem &sm,
                                           double (&acc)[XWarp<NWG>::ACC]) {
    constexpr int NT = 32 * NWG, ACC = XWarp<NWG>::ACC;
#pragma unroll
    for (int q = 0; q < ACC; ++q) acc[q] = 0.0;
    const int nk = (d.k + XBK - 1) / XBK;
    for (int kc = 0; kc < nk; ++kc) {
        cp_async_wait<XST - 2>();
        __syncthreads();
        const int nx = kc + XST - 1;
        if (nx < nk) xgemm_issue<TA, TB, NT>(d, r0, c0, nx * XBK, sm, nx % XST);
        cp_async_commit();
        xgemm_compute<TA, TB, NWG>(sm, kc % XST, acc);
    }
    cp_async_wait<0>();
    __syncthreads();  // the ring is refilled by the next tile's prologue
}

// One tile: prologue, K loop, epilogue (no overlap with a next tile).
template <int TA, int TB, int NWG = 8>
__device__ __forceinline__ void xgemm_tile(const GemmDesc &d, int r0, int c0, BigSmem &sm) {
    double acc[XWarp<NWG>::ACC];
    xgemm_prologue<TA, TB, 32 * NWG>(d, r0, c0, sm);
    xgemm_main<TA, TB, NWG>(d, r0, c0, sm, acc);
    xgemm_epilogue<NWG>(d, r0, c0, acc);
}

__device__ __forceinline__ int xgemm_tiles_of(const GemmDesc &d) {
    if (d.m <= 0 || d.n <= 0) return 0;
    return ((d.m + XBM - 1) / XBM) * ((d.n + XBN - 1) / XBN);
}
// work of one tile in units of 64 K (+1 for the epilogue)
__device__ __forceinline__ int xgemm_tile_weight(const GemmDesc &d) { return 1 + (d.k > 0 ? (d.k + 63) / 64 : 0); }

// tile_off[b] = weighted tiles before slot b (one CTA)
template <class Prob>
__global__ void __launch_bounds__(1024) xgemm_scan_kernel(Prob P, int count, const int *count_ptr, int *tile_off) {
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
            if (P.get(b, d)) v = xgemm_tiles_of(d) * xgemm_tile_weight(d);
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
            warp_sums[lane] = w;
        }
        __syncthreads();
        const int excl = carry_s + (warp ? warp_sums[warp - 1] : 0) + x - v;
        if (b < count) tile_off[b] = excl;
        __syncthreads();
        if (tid == 1023) carry_s = excl + v;
        __syncthreads();
    }
    if (tid == 0) tile_off[count] = carry_s;
}

// Persistent: CTA b owns the tiles whose weighted start lies in its 1/G share.
template <class Prob, int TA, int TB, int NWG = 8>
__global__ void __launch_bounds__(32 * NWG, XGEMM_MINB) xgemm_sched_kernel(Prob P, int count, const int *count_ptr,
                                                             const int *__restrict__ tile_off) {
    extern __shared__ __align__(16) unsigned char x_smem[];
    BigSmem &sm = *reinterpret_cast<BigSmem *>(x_smem);
    if (count < 0) count = *count_ptr;
    if (count <= 0) return;
    const int total = tile_off[count];
    const long long G = gridDim.x;
    const int u_begin = (int)((long long)blockIdx.x * total / G);
    const int u_end = (int)((long long)(blockIdx.x + 1) * total / G);
    if (u_begin >= u_end) return;
    int lo = 0, hi = count - 1;
    while (lo < hi) {
        int mid = (lo + hi + 1) >> 1;
        if (tile_off[mid] <= u_begin) lo = mid; else hi = mid - 1;
    }
    int b = lo;
    GemmDesc cur;
    P.get(b, cur);
    int w = xgemm_tile_weight(cur), off_b = tile_off[b];
    int nt_b = (tile_off[b + 1] - off_b) / w;
    int local = u_begin > off_b ? (u_begin - off_b + w - 1) / w : 0;
    // next tile of this CTA's share (false: done)
    auto advance = [&]() -> bool {
        while (local >= nt_b) {
            if (++b >= count) return false;
            off_b = tile_off[b];
            if (off_b >= u_end) return false;
            P.get(b, cur);
            w = xgemm_tile_weight(cur);
            nt_b = (tile_off[b + 1] - off_b) / w;
            local = 0;
        }
        return off_b + local * w < u_end;
    };
    if (!advance()) return;
    int ntm = (cur.m + XBM - 1) / XBM;
    int r0 = (local % ntm) * XBM, c0 = (local / ntm) * XBN;
    xgemm_prologue<TA, TB, 32 * NWG>(cur, r0, c0, sm);
    double acc[XWarp<NWG>::ACC];
    while (true) {
        xgemm_main<TA, TB, NWG>(cur, r0, c0, sm, acc);
        // the next tile's C prefetch and first K chunks go out before this
        // tile's epilogue, so their latency hides behind it
        const GemmDesc done = cur;
        const int dr0 = r0, dc0 = c0;
        ++local;
        const bool more = advance();
        if (more) {
            ntm = (cur.m + XBM - 1) / XBM;
            r0 = (local % ntm) * XBM;
            c0 = (local / ntm) * XBN;
            xgemm_prologue<TA, TB, 32 * NWG>(cur, r0, c0, sm);
        }
        xgemm_epilogue<NWG>(done, dr0, dc0, acc);
        if (!more) return;
    }
}

// ---------------------------------------------------------------------------
// Warp-specialised variant (tuning xgemm_ws = 1): the 8 DMMA warps never wait
// at a CTA barrier.  A 9th warp is the producer: it fills the 4-stage ring
// with cp.async and signals each stage's mbarrier (cp.async.mbarrier.arrive:
// the arrival fires when the copies have landed); the DMMA warps wait on the
// stage's `full` barrier, compute, and release it through its `empty`
// barrier (one arrival per warp).  The producer runs up to 4 chunks ahead,
// across tile boundaries, so the next tile's operands stream in while the
// DMMA warps run this tile's epilogue.  384 threads = 3 warpgroups launched
// at 168 registers (64,512 for the CTA); setmaxnreg moves registers from the
// producer group (56) to the DMMA groups (216) inside that allocation:
// 128 x 56 + 256 x 216 = 62,464 (an increase beyond the CTA's launch
// allocation never completes).  9 warps at 224 cannot launch at all: 3 warps
// of one SM sub-partition would need 21,504 of its 16,384 registers.
__device__ __forceinline__ unsigned smem_u32(const void *p) { return (unsigned)__cvta_generic_to_shared(p); }
__device__ __forceinline__ void mbar_init(unsigned long long *bar, unsigned count) {
    asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;\n" ::"r"(smem_u32(bar)), "r"(count) : "memory");
}
__device__ __forceinline__ void mbar_arrive(unsigned long long *bar) {
    asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];\n" ::"r"(smem_u32(bar)) : "memory");
}
__device__ __forceinline__ void mbar_arrive_cp_async(unsigned long long *bar) {
    asm volatile("cp.async.mbarrier.arrive.noinc.shared::cta.b64 [%0];\n" ::"r"(smem_u32(bar)) : "memory");
}
__device__ __forceinline__ void mbar_wait(unsigned long long *bar, unsigned parity) {
    asm volatile(
        "{\n .reg .pred p;\n"
        "XW_WAIT%=:\n"
        " mbarrier.try_wait.parity.shared::cta.b64 p, [%0], %1;\n"
        " @!p bra XW_WAIT%=;\n"
        "}\n" ::"r"(smem_u32(bar)),
        "r"(parity)
        : "memory");
}

// TMA bulk copy global -> shared, completion counted in bytes on an mbarrier
__device__ __forceinline__ void mbar_expect_tx(unsigned long long *bar, unsigned bytes) {
    asm volatile("mbarrier.expect_tx.relaxed.cta.shared::cta.b64 [%0], %1;\n" ::"r"(smem_u32(bar)), "r"(bytes)
                 : "memory");
}
__device__ __forceinline__ void bulk_g2s(void *dst, const void *src, unsigned bytes, unsigned long long *bar) {
    asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];\n" ::"r"(
                     smem_u32(dst)),
                 "l"(src), "r"(bytes), "r"(smem_u32(bar))
                 : "memory");
}
// TMA path for the A operand (TA = 0, tuning xgemm_tma): each of the 16
// k-columns of a chunk is one contiguous segment of <= 128 rows in global
// memory -> one bulk copy per column into its row of the [k][m] stage.  A
// segment that starts 8 bytes off a 16-byte boundary (odd (A + r0 + k lda))
// is copied from one element earlier, so its rows sit one slot later:
// a_shift(d, r0, k) = 1.  The extra element read before / after a segment
// stays inside the matrix: it is row c1 - 1 of the same column, or the
// element after row m - 1 of L21 column J + k, i.e. row 0 of column J + k + 1
// <= c1 < n (padding when ld > m) -- so the path is only used for the
// two-level trailing update, not for a caller's irr_gemm operands.  Only
// chunks entirely below K take this path (the K tail keeps the zero-filling
// cp.async path: A columns past K must read as zeros).
__device__ __forceinline__ int a_shift(const GemmDesc &d, int r0, int k) {
    return (int)((reinterpret_cast<uintptr_t>(d.A + r0 + (size_t)k * d.lda) >> 3) & 1);
}

constexpr int XWS_NT = 384;  // 8 DMMA warps + a producer warpgroup

template <class Prob, int TA, int TB>
__global__ void __launch_bounds__(XWS_NT, 1) xgemm_ws_kernel(Prob P, int count, const int *count_ptr,
                                                         const int *__restrict__ tile_off, int tma = 0) {
    extern __shared__ __align__(16) unsigned char x_smem[];
    BigSmem &sm = *reinterpret_cast<BigSmem *>(x_smem);
    __shared__ __align__(8) unsigned long long full_b[XST], empty_b[XST];
    if (threadIdx.x == 0) {
        for (int s = 0; s < XST; ++s) {
            mbar_init(&full_b[s], 128);  // the producer threads (cp.async arrivals)
            mbar_init(&empty_b[s], 8);  // one arrival per DMMA warp
        }
    }
    __syncthreads();
    if (count < 0) count = *count_ptr;
    if (count <= 0) return;
    const int total = tile_off[count];
    const long long G = gridDim.x;
    const int u_begin = (int)((long long)blockIdx.x * total / G);
    const int u_end = (int)((long long)(blockIdx.x + 1) * total / G);
    if (u_begin >= u_end) return;
    int lo = 0, hi = count - 1;
    while (lo < hi) {
        int mid = (lo + hi + 1) >> 1;
        if (tile_off[mid] <= u_begin) lo = mid; else hi = mid - 1;
    }
    int b = lo;
    GemmDesc cur;
    P.get(b, cur);
    int w = xgemm_tile_weight(cur), off_b = tile_off[b];
    int nt_b = (tile_off[b + 1] - off_b) / w;
    int local = u_begin > off_b ? (u_begin - off_b + w - 1) / w : 0;
    auto advance = [&]() -> bool {
        while (local >= nt_b) {
            if (++b >= count) return false;
            off_b = tile_off[b];
            if (off_b >= u_end) return false;
            P.get(b, cur);
            w = xgemm_tile_weight(cur);
            nt_b = (tile_off[b + 1] - off_b) / w;
            local = 0;
        }
        return off_b + local * w < u_end;
    };
    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    unsigned q = 0;  // chunk counter over this CTA's tiles: stage q % XST, phase (q / XST) & 1
    if (warp >= 8) {
        // ---- producer warpgroup
        asm volatile("setmaxnreg.dec.sync.aligned.u32 56;\n" ::: "memory");
        const int ptid = threadIdx.x - 256;
        while (advance()) {
            const int ntm = (cur.m + XBM - 1) / XBM;
            const int r0 = (local % ntm) * XBM, c0 = (local / ntm) * XBN;
            if (cur.beta != 0.0) {  // C tile towards L2 (4 columns x 8 lines per lane)
                for (int c = ptid; c < XBN; c += 128) {
                    if (c0 + c >= cur.n) break;
                    for (int r = 0; r < XBM; r += 16)
                        if (r0 + r < cur.m)
                            asm volatile("prefetch.global.L2 [%0];" ::"l"(cur.C + r0 + r + (size_t)(c0 + c) * cur.ldc));
                }
            }
            const int nk = (cur.k + XBK - 1) / XBK;
            for (int kc = 0; kc < nk; ++kc, ++q) {
                const int st = q % XST;
                mbar_wait(&empty_b[st], ((q / XST) & 1) ^ 1);
                const int k0 = kc * XBK;
                const bool bulk = !TA && tma && k0 + XBK <= cur.k;
                if (bulk && ptid < XBK) {
                    const int rows = imin(XBM, cur.m - r0);
                    const int sh = a_shift(cur, r0, k0 + ptid);
                    const double *src = cur.A + r0 + (size_t)(k0 + ptid) * cur.lda - sh;
                    const unsigned bytes = (unsigned)(((rows + sh) * 8 + 15) & ~15);
                    mbar_expect_tx(&full_b[st], bytes);
                    bulk_g2s(sm.A[st] + ptid * XLD_KM, src, bytes, &full_b[st]);
                }
                xgemm_issue<TA, TB, 128>(cur, r0, c0, k0, sm, st, ptid, bulk);
                mbar_arrive_cp_async(&full_b[st]);
            }
            ++local;
        }
        asm volatile("cp.async.wait_all;\n" ::: "memory");
        return;
    }
    // ---- DMMA warps
    asm volatile("setmaxnreg.inc.sync.aligned.u32 216;\n" ::: "memory");
    double acc[XWarp<8>::ACC];
    while (advance()) {
        const int ntm = (cur.m + XBM - 1) / XBM;
        const int r0 = (local % ntm) * XBM, c0 = (local / ntm) * XBN;
#pragma unroll
        for (int i = 0; i < XWarp<8>::ACC; ++i) acc[i] = 0.0;
        const int nk = (cur.k + XBK - 1) / XBK;
        for (int kc = 0; kc < nk; ++kc, ++q) {
            const int st = q % XST;
            mbar_wait(&full_b[st], (q / XST) & 1);
            // bulk-copied A columns: k = ks + (lane & 3), so the shift of a
            // lane's k-column only depends on the parity of its t
            const bool bulk = !TA && tma && kc * XBK + XBK <= cur.k;
            const int aoff = bulk ? a_shift(cur, r0, kc * XBK + (lane & 3)) : 0;
            xgemm_compute<TA, TB, 8>(sm, st, acc, aoff);
            __syncwarp();
            if (lane == 0) mbar_arrive(&empty_b[st]);
        }
        xgemm_epilogue<8>(cur, r0, c0, acc);
        ++local;
    }
}

// Wraps a problem and keeps only the slots one of the two cores should run:
// the big core takes products whose tile would be mostly full and whose K
// amortises the pipeline fill.
template <class Prob>
struct SizeFilter {
    Prob p;
    int want_big;
    __device__ static bool is_big(const GemmDesc &d) { return d.m >= 96 && d.n >= 96 && d.k >= 48; }
    __device__ bool get(int slot, GemmDesc &d) const {
        if (!p.get(slot, d)) return false;
        if (want_big >= 0 && is_big(d) != (want_big != 0)) { d.m = 0; d.n = 0; d.k = 0; return false; }
        return true;
    }
};

template <class Prob, int TA, int TB>
inline void xgemm_launch_t(const Prob &P, int cnt, const int *cnt_ptr, const int *tile_off, cudaStream_t s) {
    if (tuning().xgemm_warps == 9) {
        smem_optin(xgemm_ws_kernel<Prob, TA, TB>, BIG_SMEM);
        // no TMA path here: a caller's A may end (or start) exactly at its
        // allocation, and a shifted / rounded segment reads 8 bytes past it
        xgemm_ws_kernel<Prob, TA, TB><<<num_sms(), XWS_NT, BIG_SMEM, s>>>(P, cnt, cnt_ptr, tile_off, 0);
        return;
    }
    smem_optin(xgemm_sched_kernel<Prob, TA, TB>, BIG_SMEM);
    xgemm_sched_kernel<Prob, TA, TB><<<num_sms() * XGEMM_MINB, X_NT, BIG_SMEM, s>>>(P, cnt, cnt_ptr, tile_off);
}

// one persistent CTA per SM; the transposes select the shared layouts
template <class Prob>
inline void launch_xgemm(const Prob &P, int ta, int tb, int cnt, const int *cnt_ptr, const int *tile_off,
                         cudaStream_t s) {
    if (!ta && !tb) xgemm_launch_t<Prob, 0, 0>(P, cnt, cnt_ptr, tile_off, s);
    else if (!ta && tb) xgemm_launch_t<Prob, 0, 1>(P, cnt, cnt_ptr, tile_off, s);
    else if (ta && !tb) xgemm_launch_t<Prob, 1, 0>(P, cnt, cnt_ptr, tile_off, s);
    else xgemm_launch_t<Prob, 1, 1>(P, cnt, cnt_ptr, tile_off, s);
}

}  // namespace irr

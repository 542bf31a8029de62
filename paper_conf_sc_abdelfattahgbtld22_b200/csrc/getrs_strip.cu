// getrs_strip.cu -- step a5.2 of the partial front factorization (SURVEY
// §8(a)), F12 <- U11^-1 L11^-1 P^T F12, as ONE kernel.
//
// The paper composes this step from irrLASWP + two irrTRSM calls (P:L96,
// L175-182).  On a multifrontal batch the recursive TRSM needs a launch chain
// per level and per leaf (the host drives the recursion), and the
// row interchanges walk every column of F12 once per pivot block.  Here the
// work unit is a (front, 64-column strip of F12): the strip's columns belong
// to one CTA for the whole step, so the step has no inter-CTA dependency at
// all and a single launch covers the batch:
//   1. P^T: the n1 interchanges are composed into a gather permutation in
//      shared memory (the "rehearsal" of P:L192, serial over n1 on one
//      thread), then each column of the strip is read once, permuted in
//      shared memory and written once (coalesced both ways);
//   2. L^-1 (unit lower) and 3. U^-1 (non-unit upper), blocked by 64 rows,
//      left-looking: block I of the strip is first updated with the already
//      solved blocks, X_I -= T(I, done) X(done), on the FP64 tensor core
//      (mma.sync DMMA m8n8k4, 64 x 64 tile, 8 warps of 32 x 16), then solved
//      against the 64 x 64 diagonal triangle by substitution in registers
//      (4 lanes per column, 16 interleaved rows each, x_s by shuffle).  No explicit
//      inverse; the diagonal of U divides, as the oracle does.
// The strip stays in F12 (L2-resident while its CTA works on it).
#include "gemm_core.cuh"
#include "sched.cuh"

namespace irr {

#ifndef IRR_GS_SW
#define IRR_GS_SW 64
#endif
// strip width (right-hand sides per unit), 64 or 128 (build switch): 128
// halves the re-reads of F11 per front and gives each warp a 32 x 32 tile,
// but needs a 3-deep ring for 2 CTAs / SM and was measured slower (C4 a5.2
// 30.15 vs 29.33 ms, profiles/r02/s2/r3m_*)
constexpr int GS_SW = IRR_GS_SW;
constexpr int GS_NI = GS_SW / 32;  // 8-column DMMA tiles per warp (warps: 2 along m x 4 along n)
constexpr int GS_CPQ = GS_SW / 64; // columns per 4-lane group in the substitution
constexpr int GS_BR = 64;     // row block of the blocked solve
constexpr int GS_NT = 256;
constexpr int GS_BK = 16;     // K chunk of the update GEMM
constexpr int GS_ST = GS_SW > 64 ? 3 : 4;  // cp.async ring depth (2 CTAs / SM must fit)
constexpr int GS_LDA = GS_BR + 4;  // [k][m] layout, conflict-free fragments
constexpr int GS_LDB = GS_BK + 4;  // [n][k] layout
constexpr int GS_LDT = GS_BR + 1;
constexpr int GS_N1MAX = 4096;

struct GsRing {
    double A[GS_ST][GS_BK * GS_LDA];
    double B[GS_ST][GS_SW * GS_LDB];
};
struct GsSolve {
    double T[GS_BR * GS_LDT];  // diagonal triangle, column-major
    double X[GS_SW * GS_LDT];  // the block being solved: X[c * GS_LDT + r]
    double rd[GS_BR];          // upper solve: reciprocals of the diagonal
};
// The ring (update GEMM) and the solve buffers are used one after the other
// and share the same bytes; the permutation phase (perm + ipiv ints and a
// two-column buffer) comes first and shares them too.
constexpr size_t GS_PERM_BYTES = 2 * GS_N1MAX * sizeof(int) + 2 * GS_N1MAX * sizeof(double);
constexpr size_t GS_SOLVE_BYTES = sizeof(GsRing) > sizeof(GsSolve) ? sizeof(GsRing) : sizeof(GsSolve);
constexpr size_t GS_SMEM = GS_PERM_BYTES > GS_SOLVE_BYTES ? GS_PERM_BYTES : GS_SOLVE_BYTES;

struct GsArgs {
    int batch;
    const int *n1, *n2;
    const double *const *F11; const int *ld11;
    double *const *F12; const int *ld12;
    int *const *ipiv;
    const int *info;  // fronts with info < 0 (bad arguments) are skipped
    int upper;        // 0: stop after L^-1 (U12 of the LAPACK-style partial)
};

struct GsUnits {
    GsArgs g;
    __device__ int units(int i) const {
        const int a = g.n1[i], b = g.n2[i];
        if (a <= 0 || b <= 0 || g.info[i] < 0) return 0;
        return (b + GS_SW - 1) / GS_SW;
    }
};

// ---- the update GEMM: acc (64 x 64 tile of the strip, fragment layout)
//      -= T(rows r0.., cols k0..k0+K) * X(rows k0..k0+K, strip)
__device__ __forceinline__ void gs_issue(const double *T, long ldt, int r0, int rb, const double *X, long ldx,
                                         int c0, int W, int kbeg, int k0, int kend, GsRing &rg, int st) {
    // pairs of consecutive elements (rows of T, k of X): one 16-byte copy
    // where the pair is aligned in global memory, else two 8-byte copies
    // (ncu: the per-element copies were ~10% of the kernel's stall samples)
    const int tid = threadIdx.x;
#pragma unroll
    for (int q = 0; q < (GS_BR * GS_BK) / (2 * GS_NT); ++q) {
        const int e = tid + GS_NT * q;
        const int m = 2 * (e & (GS_BR / 2 - 1)), kk = e / (GS_BR / 2);
        const int gk = k0 + kk;
        double *dst = &rg.A[st][kk * GS_LDA + m];
        const double *src = T + r0 + m + (size_t)gk * ldt;
        const bool okk = gk < kend;
        if (okk && m + 1 < rb && ((reinterpret_cast<uintptr_t>(src) & 15) == 0)) {
            cp_async16(dst, src);
        } else {
            if (okk && m < rb) cp_async8(dst, src); else dst[0] = 0.0;
            if (okk && m + 1 < rb) cp_async8(dst + 1, src + 1); else dst[1] = 0.0;
        }
    }
#pragma unroll
    for (int q = 0; q < (GS_SW * GS_BK) / (2 * GS_NT); ++q) {
        const int e = tid + GS_NT * q;
        const int kk = 2 * (e & (GS_BK / 2 - 1)), n = e / (GS_BK / 2);
        const int gk = k0 + kk;
        double *dst = &rg.B[st][n * GS_LDB + kk];
        const double *src = X + gk + (size_t)(c0 + n) * ldx;
        const bool okn = n < W;
        if (okn && gk + 1 < kend && ((reinterpret_cast<uintptr_t>(src) & 15) == 0)) {
            cp_async16(dst, src);
        } else {
            if (okn && gk < kend) cp_async8(dst, src); else dst[0] = 0.0;
            if (okn && gk + 1 < kend) cp_async8(dst + 1, src + 1); else dst[1] = 0.0;
        }
    }
    (void)kbeg;
}

__device__ __forceinline__ void gs_update(double (&acc)[8 * GS_NI], const double *T, long ldt, int r0, int rb,
                                          const double *X, long ldx, int c0, int W, int kbeg, int kend, GsRing &rg) {
    if (kend <= kbeg) return;
    const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
    const int g = lane >> 2, t = lane & 3;
    const int wm = (warp & 1) * 32, wn = (warp >> 1) * (8 * GS_NI);
    const int nk = (kend - kbeg + GS_BK - 1) / GS_BK;
#pragma unroll
    for (int st = 0; st < GS_ST - 1; ++st) {
        if (st < nk) gs_issue(T, ldt, r0, rb, X, ldx, c0, W, kbeg, kbeg + st * GS_BK, kend, rg, st);
        cp_async_commit();
    }
    for (int kc = 0; kc < nk; ++kc) {
        cp_async_wait<GS_ST - 2>();
        __syncthreads();
        const int nx = kc + GS_ST - 1;
        if (nx < nk) gs_issue(T, ldt, r0, rb, X, ldx, c0, W, kbeg, kbeg + nx * GS_BK, kend, rg, nx % GS_ST);
        cp_async_commit();
        const double *As = rg.A[kc % GS_ST];
        const double *Bs = rg.B[kc % GS_ST];
#pragma unroll
        for (int ks = 0; ks < GS_BK; ks += 4) {
            double a[4], b[GS_NI];
#pragma unroll
            for (int mi = 0; mi < 4; ++mi) a[mi] = -As[(ks + t) * GS_LDA + wm + 8 * mi + g];
#pragma unroll
            for (int ni = 0; ni < GS_NI; ++ni) b[ni] = Bs[(wn + 8 * ni + g) * GS_LDB + ks + t];
#pragma unroll
            for (int mi = 0; mi < 4; ++mi)
#pragma unroll
                for (int ni = 0; ni < GS_NI; ++ni) {
                    // acc -= a b : one operand negated (exact)
                    dmma_8x8x4(acc[(mi * GS_NI + ni) * 2], acc[(mi * GS_NI + ni) * 2 + 1], a[mi], b[ni]);
                }
        }
    }
    cp_async_wait<0>();
    __syncthreads();  // the ring's bytes are reused by the solve buffers
}

// ---- one 64-row block: load X_I into the accumulators, update, stage in smem,
//      solve against the diagonal triangle, write back.  lower: unit lower
//      forward substitution; else non-unit upper backward substitution.
template <bool LOWER>
__device__ __forceinline__ void gs_block(const double *T, long ldt, double *X, long ldx, int n1, int c0, int W,
                                         int r0, GsRing &rg, GsSolve &sv) {
    const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
    const int g = lane >> 2, t = lane & 3;
    const int wm = (warp & 1) * 32, wn = (warp >> 1) * (8 * GS_NI);
    const int rb = imin(GS_BR, n1 - r0);
    double acc[8 * GS_NI];
#pragma unroll
    for (int mi = 0; mi < 4; ++mi)
#pragma unroll
        for (int ni = 0; ni < GS_NI; ++ni)
#pragma unroll
            for (int i = 0; i < 2; ++i) {
                const int r = wm + 8 * mi + g, c = wn + 8 * ni + 2 * t + i;
                acc[(mi * GS_NI + ni) * 2 + i] = (r < rb && c < W) ? X[r0 + r + (size_t)(c0 + c) * ldx] : 0.0;
            }
    if (LOWER) gs_update(acc, T, ldt, r0, rb, X, ldx, c0, W, 0, r0, rg);
    else gs_update(acc, T, ldt, r0, rb, X, ldx, c0, W, r0 + rb, n1, rg);
    // the diagonal triangle (into the ring's bytes, now free)
    for (int e = tid; e < GS_BR * GS_BR; e += GS_NT) {
        const int r = e & (GS_BR - 1), c = e >> 6;
        double *dst = &sv.T[c * GS_LDT + r];
        if (r < rb && c < rb) cp_async8(dst, T + r0 + r + (size_t)(r0 + c) * ldt);
        else *dst = (r == c) ? 1.0 : 0.0;
    }
    cp_async_commit();
    // accumulators -> shared X block
#pragma unroll
    for (int mi = 0; mi < 4; ++mi)
#pragma unroll
        for (int ni = 0; ni < GS_NI; ++ni)
#pragma unroll
            for (int i = 0; i < 2; ++i) {
                const int r = wm + 8 * mi + g, c = wn + 8 * ni + 2 * t + i;
                sv.X[c * GS_LDT + r] = acc[(mi * GS_NI + ni) * 2 + i];
            }
    cp_async_wait<0>();
    __syncthreads();
    if (!LOWER) {
        // one true division per diagonal entry, then multiplies in the
        // substitution (ncu: the per-step division was 14% of the kernel's
        // stall samples and 13% of its instructions)
        if (tid < GS_BR) sv.rd[tid] = 1.0 / sv.T[tid * GS_LDT + tid];
        __syncthreads();
    }
    // substitution: columns c = tid >> 2 (and c + 64 when the strip is 128
    // wide, one after the other: two live chains spill at 128 registers);
    // lane q4 = tid & 3 owns rows q4 + 4k (interleaved, so the four lanes of
    // a column read four consecutive T entries: conflict-free); x_s comes
    // from lane s & 3 by shuffle
#pragma unroll 1
    for (int h = 0; h < GS_CPQ; ++h) {
        const int c = (tid >> 2) + 64 * h, q4 = tid & 3;
        const int base = lane & ~3;
        double x[16];
#pragma unroll
        for (int k = 0; k < 16; ++k) x[k] = sv.X[c * GS_LDT + q4 + 4 * k];
        // steps in chunks of 16 (compile-time register index), only as many
        // chunks as the block has rows (rows >= rb are zero and stay zero)
        if (LOWER) {
#pragma unroll
            for (int s0 = 0; s0 < GS_BR; s0 += 16) {
                if (s0 >= rb) break;
#pragma unroll
                for (int ss = 0; ss < 16; ++ss) {
                    const int s = s0 + ss;
                    const double xs = __shfl_sync(FULL, x[s >> 2], base | (s & 3));
                    const double *Ts = sv.T + s * GS_LDT + q4;
#pragma unroll
                    for (int k = s >> 2; k < 16; ++k)
                        if (q4 + 4 * k > s) x[k] = fma(-Ts[4 * k], xs, x[k]);
                }
            }
        } else {
#pragma unroll
            for (int s0 = GS_BR - 16; s0 >= 0; s0 -= 16) {
                if (s0 >= rb) continue;
#pragma unroll
                for (int ss = 15; ss >= 0; --ss) {
                    const int s = s0 + ss;
                    if (q4 == (s & 3)) x[s >> 2] = x[s >> 2] * sv.rd[s];
                    const double xs = __shfl_sync(FULL, x[s >> 2], base | (s & 3));
                    const double *Ts = sv.T + s * GS_LDT + q4;
#pragma unroll
                    for (int k = 0; k <= (s >> 2); ++k)
                        if (q4 + 4 * k < s) x[k] = fma(-Ts[4 * k], xs, x[k]);
                }
            }
        }
        if (c < W) {
#pragma unroll
            for (int k = 0; k < 16; ++k)
                if (q4 + 4 * k < rb) X[r0 + q4 + 4 * k + (size_t)(c0 + c) * ldx] = x[k];
        }
    }
    __syncthreads();  // X block visible to the next block's update; smem reusable
}

// Units are handed out by an atomic queue in the order of the size sort
// (largest n1 first): a strip of a 2000-row front is ~1000x the work of one
// of a 30-row front, so equal unit counts per CTA would leave a dozen CTAs
// holding every large front.
__global__ void __launch_bounds__(GS_NT, 2) getrs_strip_kernel(GsArgs g, SlotList sl, const int *units_off,
                                                               int *queue) {
    extern __shared__ __align__(16) unsigned char gs_smem[];
    GsRing &rg = *reinterpret_cast<GsRing *>(gs_smem);
    GsSolve &sv = *reinterpret_cast<GsSolve *>(gs_smem);
    int *perm = reinterpret_cast<int *>(gs_smem);
    int *ipv = perm + GS_N1MAX;
    double *colbuf = reinterpret_cast<double *>(ipv + GS_N1MAX);
    const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
    __shared__ int unit_s, slot_s;
    const int count = sl.count(g.batch);
    const int total = count > 0 ? units_off[count] : 0;
    auto body = [&](int i, int q) {
        const int n1 = g.n1[i], n2 = g.n2[i];
        const int c0 = q * GS_SW, W = imin(GS_SW, n2 - c0);
        const long ld11 = g.ld11[i], ld12 = g.ld12[i];
        const double *F11 = g.F11[i];
        double *X = g.F12[i];
        // ---- 1. P^T on the strip: compose the interchanges, permute each column
        {
            const int *ip = g.ipiv[i];
            for (int r = tid; r < n1; r += GS_NT) { perm[r] = r; ipv[r] = ip[r] - 1; }
            __syncthreads();
            if (tid == 0) {
                for (int k = 0; k < n1; ++k) {
                    const int p = ipv[k];
                    if (p != k) {
                        const int x = perm[k];
                        perm[k] = perm[p];
                        perm[p] = x;
                    }
                }
            }
            __syncthreads();
            bool moved = false;
            for (int r = tid; r < n1; r += GS_NT) moved |= perm[r] != r;
            if (__syncthreads_or(moved)) {
                // as many columns per round as the buffer holds (was 2: the
                // rounds' load latency was ~20% of the kernel's stall samples)
                constexpr int CAP = (int)((GS_SMEM - 2 * GS_N1MAX * sizeof(int)) / sizeof(double));
                const int per = imax(1, imin(W, CAP / n1));
                for (int cc = 0; cc < W; cc += per) {
                    const int nc = imin(per, W - cc);
                    for (int c = warp; c < nc; c += GS_NT / 32) {
                        const double *col = X + (size_t)(c0 + cc + c) * ld12;
                        for (int r = lane; r < n1; r += 32) cp_async8(&colbuf[(size_t)c * n1 + r], col + r);
                    }
                    cp_async_commit();
                    cp_async_wait<0>();
                    __syncthreads();
                    for (int c = warp; c < nc; c += GS_NT / 32) {
                        double *col = X + (size_t)(c0 + cc + c) * ld12;
                        for (int r = lane; r < n1; r += 32) {
                            const int p = perm[r];
                            if (p != r) col[r] = colbuf[(size_t)c * n1 + p];
                        }
                    }
                    __syncthreads();
                }
            }
        }
            // ---- 2. L^-1 (unit lower), blocks top to bottom
        for (int r0 = 0; r0 < n1; r0 += GS_BR) gs_block<true>(F11, ld11, X, ld12, n1, c0, W, r0, rg, sv);
        // ---- 3. U^-1 (non-unit upper), blocks bottom to top
        if (!g.upper) return;
        const int last = ((n1 - 1) / GS_BR) * GS_BR;
        for (int r0 = last; r0 >= 0; r0 -= GS_BR) gs_block<false>(F11, ld11, X, ld12, n1, c0, W, r0, rg, sv);
    };
    while (true) {
        if (tid == 0) {
            const int u = atomicAdd(queue, 1);
            int b = -1;
            if (u < total) {
                int lo = 0, hi = count - 1;  // last slot with units_off[slot] <= u
                while (lo < hi) {
                    const int mid = (lo + hi + 1) >> 1;
                    if (units_off[mid] <= u) lo = mid; else hi = mid - 1;
                }
                b = lo;
            }
            unit_s = u;
            slot_s = b;
        }
        __syncthreads();
        const int u = unit_s, b = slot_s;
        __syncthreads();
        if (b < 0) break;
        body(sl.matrix(b), u - units_off[b]);
    }
}

// true when the fused kernel can take the step (n1 fits the permutation buffer)
bool getrs_strip_ok(int max_n1) { return max_n1 <= GS_N1MAX; }

void launch_getrs_strip(int batch, const int *n1, const int *n2, const double *const *F11, const int *ld11,
                        double *const *F12, const int *ld12, int *const *ipiv, const int *info, int *units_off,
                        int *queue, SlotList sl, cudaStream_t s, int upper) {
    GsArgs g{batch, n1, n2, F11, ld11, F12, ld12, ipiv, info, upper};
    smem_optin(getrs_strip_kernel, GS_SMEM);
    {
        KScope k(K_GEMM_SCAN, s);
        scan_units_kernel<GsUnits><<<1, 1024, 0, s>>>(GsUnits{g}, sl, batch, units_off);
    }
    cudaMemsetAsync(queue, 0, sizeof(int), s);
    KScope k(K_GETRS, s);
    getrs_strip_kernel<<<num_sms() * 2, GS_NT, GS_SMEM, s>>>(g, sl, units_off, queue);
}

}  // namespace irr

// Batched extend-add: child Schur complements scattered into their parent
// fronts (§III-A "the Schur complement F_{r:22} is added into the
// parent frontal matrix ... this requires a scatter operation"; L102: every
// front of one tree level at once).  include/irr.h irr_extend_add.
//
// HBM-bound scatter: 8 B read of F22 + one 8 B FP64 reduction (RED.ADD.F64,
// resolved in L2, fire-and-forget) per child element, plus the parent entry's
// read-modify-write in L2.  No tensor-core work.  Layout:
//   * grid.x = child, grid.y splits the child's columns (j = y, y + Y, ...);
//   * the CTA's columns are flattened with the rows so that tiny children
//     (n2 < 256) still keep every thread busy; along a column consecutive
//     threads read consecutive F22 rows (coalesced) and write rel-mapped rows
//     of the same parent column (sorted rel => mostly the same sectors);
//   * rel is staged once per CTA in shared memory (first EA_REL_SMEM entries)
//     and validated there (one __syncthreads_or), so a bad map adds nothing.
#include "irr_internal.cuh"

namespace irr {

constexpr int EA_THREADS = 256;
constexpr int EA_REL_SMEM = 4096;  // 16 KB of rel entries per CTA
constexpr int EA_MAX_Y = 64;
#ifndef EA_PER_CTA
#define EA_PER_CTA 16384  // target child elements per CTA of the largest child
#endif

// fire-and-forget FP64 reduction (atomicAdd with an unused result compiles to
// ATOM, whose return the warp waits for: 88% long-scoreboard stalls in ncu)
__device__ __forceinline__ void red_add_f64(double *p, double v) {
    asm volatile("red.relaxed.gpu.global.add.f64 [%0], %1;" ::"l"(p), "d"(v) : "memory");
}

__global__ void __launch_bounds__(EA_THREADS)
    extend_add_kernel(int max_n2, const int *__restrict__ n2, const double *const *__restrict__ F22,
                      const int *__restrict__ ld22, const int *const *__restrict__ rel, const int *__restrict__ np,
                      double *const *__restrict__ Fp, const int *__restrict__ ldp, int *__restrict__ info) {
    __shared__ int srel[EA_REL_SMEM];
    const int c = blockIdx.x;
    const int nc = n2[c], npc = np[c], l22 = ld22[c], lp = ldp[c];
    int code = 0;
    if (nc < 0 || nc > max_n2) code = -3;
    else if (l22 < max(1, nc)) code = -5;
    else if (npc < 0) code = -7;
    else if (lp < max(1, npc)) code = -9;
    else if (nc > 0 && !F22[c]) code = -4;
    else if (nc > 0 && !Fp[c]) code = -8;
    else if (nc > 0 && !rel[c]) code = -6;
    if (code != 0 || nc == 0) {
        if (blockIdx.y == 0 && threadIdx.x == 0) info[c] = code;
        return;
    }
    const int *r = rel[c];
    int bad = 0;
    for (int i = threadIdx.x; i < nc; i += EA_THREADS) {
        int v = __ldg(r + i);
        if (i < EA_REL_SMEM) srel[i] = v;
        bad |= (v < 0 || v >= npc);
    }
    bad = __syncthreads_or(bad);
    if (blockIdx.y == 0 && threadIdx.x == 0) info[c] = bad ? -6 : 0;
    if (bad) return;

    const int Y = gridDim.y;
    if ((int)blockIdx.y >= nc) return;
    const int ncols = (nc - (int)blockIdx.y + Y - 1) / Y;  // columns j = y + q*Y, q < ncols
    const long long total = (long long)ncols * nc;
    const double *A = F22[c];
    double *P = Fp[c];
    // walk (i, q) in column-major order without a division per element
    long long e = threadIdx.x;
    int q = (int)(e / nc), i = (int)(e - (long long)q * nc);
    const int dq = EA_THREADS / nc, di = EA_THREADS - dq * nc;  // step of EA_THREADS elements
    for (; e < total; e += EA_THREADS) {
        const int j = (int)blockIdx.y + q * Y;
        const int ri = i < EA_REL_SMEM ? srel[i] : __ldg(r + i);
        const int rj = j < EA_REL_SMEM ? srel[j] : __ldg(r + j);
        const double v = __ldg(A + (size_t)i + (size_t)j * l22);
        red_add_f64(P + (size_t)ri + (size_t)rj * lp, v);
        i += di;
        q += dq;
        if (i >= nc) {
            i -= nc;
            ++q;
        }
    }
}

// Small children (max_n2 <= 64): one warp per child, 8 children per CTA, rel
// held in two registers per lane and broadcast by shuffles -- no shared
// memory stage and no CTA barrier per child (the CTA-per-child kernel spends
// its time on that prologue when a child has only a few hundred elements).
constexpr int EA_SMALL_N2 = 64;
__global__ void __launch_bounds__(256)
    extend_add_small_kernel(int batch, int max_n2, const int *__restrict__ n2, const double *const *__restrict__ F22,
                            const int *__restrict__ ld22, const int *const *__restrict__ rel,
                            const int *__restrict__ np, double *const *__restrict__ Fp, const int *__restrict__ ldp,
                            int *__restrict__ info) {
    const int lane = threadIdx.x & 31;
    const int c = blockIdx.x * 8 + (threadIdx.x >> 5);
    if (c >= batch) return;
    const int nc = n2[c], npc = np[c], l22 = ld22[c], lp = ldp[c];
    int code = 0;
    if (nc < 0 || nc > max_n2) code = -3;
    else if (l22 < max(1, nc)) code = -5;
    else if (npc < 0) code = -7;
    else if (lp < max(1, npc)) code = -9;
    else if (nc > 0 && !F22[c]) code = -4;
    else if (nc > 0 && !Fp[c]) code = -8;
    else if (nc > 0 && !rel[c]) code = -6;
    if (code != 0 || nc == 0) {
        if (lane == 0) info[c] = code;
        return;
    }
    const int *r = rel[c];
    const int r0 = lane < nc ? __ldg(r + lane) : 0;
    const int r1 = lane + 32 < nc ? __ldg(r + lane + 32) : 0;
    const bool bad = __any_sync(0xffffffffu, r0 < 0 || r0 >= npc || r1 < 0 || r1 >= npc);
    if (lane == 0) info[c] = bad ? -6 : 0;
    if (bad) return;
    const double *A = F22[c];
    double *P = Fp[c];
    const int total = nc * nc;
    int j = lane / nc, i = lane - j * nc;
    const int dj = 32 / nc, di = 32 - dj * nc;
    for (int e = lane; e - lane < total; e += 32) {  // whole warp iterates (shuffles)
        const int a0 = __shfl_sync(0xffffffffu, r0, i & 31), a1 = __shfl_sync(0xffffffffu, r1, i & 31);
        const int b0 = __shfl_sync(0xffffffffu, r0, j & 31), b1 = __shfl_sync(0xffffffffu, r1, j & 31);
        if (e < total) {
            const int ri = i < 32 ? a0 : a1, rj = j < 32 ? b0 : b1;
            red_add_f64(P + (size_t)ri + (size_t)rj * lp, __ldg(A + (size_t)i + (size_t)j * l22));
        }
        i += di;
        j += dj;
        if (i >= nc) {
            i -= nc;
            ++j;
        }
    }
}

void launch_extend_add(int batch, int max_n2, const int *n2, const double *const *F22, const int *ld22,
                       const int *const *rel, const int *np, double *const *Fp, const int *ldp, int *info,
                       cudaStream_t s) {
    // about 16 K elements per CTA of the largest child, at most EA_MAX_Y column groups
    long long per = (long long)max_n2 * max_n2;
    int Y = (int)std::min<long long>(EA_MAX_Y, std::max<long long>(1, (per + EA_PER_CTA - 1) / EA_PER_CTA));
    Y = std::max(1, std::min(Y, std::max(1, max_n2)));
    KScope k(K_EXTEND_ADD, s);
    if (max_n2 <= EA_SMALL_N2) {
        extend_add_small_kernel<<<(batch + 7) / 8, 256, 0, s>>>(batch, max_n2, n2, F22, ld22, rel, np, Fp, ldp, info);
        return;
    }
    extend_add_kernel<<<dim3(batch, Y), EA_THREADS, 0, s>>>(max_n2, n2, F22, ld22, rel, np, Fp, ldp, info);
}

}  // namespace irr

// irr_internal.cuh -- device/host internals shared by the libirr kernels.
// (Product code only; the CPU oracle under oracle/ shares nothing with this.)
#pragma once

#include <cuda_runtime.h>
#include <stdint.h>
#include <float.h>

#include "irr.h"

namespace irr {

constexpr unsigned FULL = 0xffffffffu;

// ---------------------------------------------------------------- tuning
struct Tuning {
    int nb;          // tier-L panel width ("typically 16-32 columns")
    int tier_s;      // 1: warp-per-matrix tier for m, n <= 32; 2: + several matrices per warp for m, n <= 16
    int tier_m_max;  // max padded m*n (doubles) of the shared-memory tier
    int panel_rows;  // max rows of a tier-L panel staged in shared memory
    int trsm_nb;     // TRSM recursion leaf (<= 32)
    int l1;          // 1: CTA-per-matrix tier for tier-L matrices with m <= L1_MAX_ROWS
    int phase_timing;  // 1: accumulate per-phase SM cycles into the workspace counters
    int l1_ctas_per_sm;  // resident CTAs per SM of the L1 kernel (1..3)
    int concurrent;      // 1: tiers S/M on a forked stream, concurrent with L1/L2
    int dmma;            // 1: grid-wide GEMMs on the FP64 tensor core (mma.sync DMMA), 0: DFMA
    int l1_dmma;         // same switch for the GEMM phase inside the L1 kernel
    int panel_win;       // 1: grid-wide panels by the windowed register panel (rows <= 2048)
    int strip;           // 1: fused interchange + TRSM + GEMM per 64-column strip (needs panel_win)
    int gemm_big;        // 1: long-K DCWI GEMMs on the 128x128 DMMA core (gemm_big.cuh)
    int unused_;         // (was: row-map L1 variant, measured slower in round 1, removed)
    int getrs_fused;     // 1: partial-front step a5.2 by the fused strip kernel (getrs_strip.cu)
    int l1_rows;         // max rows of the CTA-per-matrix tier (<= L1_TALL_ROWS)
    int defer;           // 1: left-block interchanges applied once at the end, coalesced (L1 and grid tiers)
    int getrs_vec;       // 1: irr_getrs with max_nrhs <= 4 by the CTA-per-system kernel (getrs_vec.cu)
    int nb_outer;        // grid-wide tier: outer block width of the two-level blocking (0 / <= nb: one level)
    int xgemm_warps;     // 8 or 16 warps per 128 x 128 DMMA tile CTA, or 9 = 8 DMMA warps + 1 producer warp (mbarrier ring)
    int parts;           // two-level grid tier: 1, or 2 halves of the LPT list on two streams
    int part_grid;       // with 2 parts: 1 = full grids per part, 2 = half grids
    int outer_cols;      // two-level interchange + U12 solve strip width: 64 (L11 square, 1 CTA/SM) or 32 (packed, 2/SM)
    int xgemm_tma;       // warp-specialised xgemm: A operand (K-chunk columns) by TMA bulk copies (cp.async.bulk)
    int mid_dmma;        // tier M: trailing update in shared memory on the FP64 tensor core (mma.sync DMMA)
    int split_strip;     // two-level inner steps: 1 = trailing update as a grid-wide GEMM, 2 = auto (few matrices)
};
Tuning &tuning();

// host-side launch counter (per thread)
long long &launch_counter();
inline void count_launch(int k = 1) { launch_counter() += k; }

// kernel classes for the optional per-class device timing (irr_profile_*)
enum KClass {
    K_CLASSIFY = 0, K_LU_SMALL, K_LU_MID, K_PANEL, K_SWAP_TRSM, K_GEMM_SCAN, K_GEMM_TRAIL,
    K_TRSM_LEAF, K_GEMM_DCWI, K_LASWP, K_MISC, K_LU_L1, K_STRIP, K_GETRS, K_EXTEND_ADD, K_ZGETRF, K_OUTER_TRSM, K_LEFT_SWAPS, NKCLASS
};
void prof_record(int cls, cudaStream_t s, bool begin);
bool prof_on();
// RAII scope around one kernel launch: counts it and, when profiling is on,
// brackets it with CUDA events on its stream.
struct KScope {
    int cls;
    cudaStream_t s;
    KScope(int c, cudaStream_t st) : cls(c), s(st) {
        if (prof_on()) prof_record(cls, s, true);
    }
    ~KScope() {
        if (prof_on()) prof_record(cls, s, false);
        count_launch();
    }
};

// ---------------------------------------------------------------- bins
// Size classes of irr_getrf (a pure function of (m_i, n_i), SURVEY §7 hard
// part 7): S = warp per matrix; M1..M3 = CTA per matrix with the whole matrix
// in shared memory (three footprints so small ones pack several CTAs per SM);
// L = blocked right-looking LU with one kernel chain per panel iteration.
// L1 = tier L with m <= L1_MAX_ROWS, one CTA per matrix; L = the rest, grid-wide
// kernels per panel iteration.
enum Bin { BIN_S = 0, BIN_M1 = 1, BIN_M2 = 2, BIN_M3 = 3, BIN_L = 4, BIN_L1 = 5, BIN_S16 = 6, BIN_S8 = 7, BIN_L1T = 8,
           BIN_S16G = 9, BIN_S8G = 10, BIN_S24 = 11, NBINS = 12 };
// L1T: CTA-per-matrix tier, 257..l1_rows rows (tall-panel kernel variant);
// S16G / S8G: m, n <= 16 / 8, several matrices per warp; S24: m <= 32, 16 < n <= 24
// on its own register budget (tuning tier_s = 2)
constexpr int L1_MAX_ROWS = 256;    // panels up to this many rows are staged in shared memory
constexpr int L1_TALL_ROWS = 1024;  // taller L1 panels: panel_win in global memory (128 threads x 8 rows)
constexpr int M1_ELEMS = 6144;    // 48 KB  -> 4 CTAs / SM
constexpr int M2_ELEMS = 12288;   // 96 KB  -> 2 CTAs / SM
constexpr int TIER_M_MAX_DEFAULT = 24576;  // 192 KB -> 1 CTA / SM

// shared-memory leading dimension of a tier-M matrix: odd, so row-wise
// accesses of consecutive columns fall in different banks
__host__ __device__ inline int mid_lds(int m) { return m | 1; }

// counters block at the head of every workspace (ints)
constexpr int CNT_INTS = 64;
enum CounterSlot { CNT_BIN0 = 48 /* NBINS ints */, CNT_MAXM = 9, CNT_MAXN = 10, CNT_L1_NEXT = 11, CNT_STRIPQ = 12, CNT_GSQ = 13, CNT_LSWQ = 14, CNT_OUTQ = 15, CNT_ZQ = 16, CNT_PANELQ = 17,
                   CNT_PHASE0 = 32 /* 8 x u64 phase-cycle accumulators (tuning phase_timing) */ };
static_assert(CNT_BIN0 + NBINS <= CNT_INTS && CNT_PHASE0 + 16 <= CNT_BIN0, "counter slots overlap");

inline size_t align256(size_t x) { return (x + 255) & ~size_t(255); }

// ---------------------------------------------------------------- device helpers
__device__ __forceinline__ unsigned long long dkey(double absv) {
    return (unsigned long long)__double_as_longlong(absv);
}

// Warp arg-max of (key, row) over lanes with cand == true: the largest key,
// ties -> the smallest row (BLAS idamax).  Keys are the bit
// patterns of non-negative doubles, so integer order == value order.
// Returns row = -1 if no lane is a candidate.
__device__ __forceinline__ void warp_argmax(bool cand, unsigned long long key, int row,
                                            unsigned long long &kout, int &rout) {
    unsigned hi = cand ? (unsigned)(key >> 32) : 0u;
    unsigned lo = cand ? (unsigned)(key & 0xffffffffu) : 0u;
    unsigned mhi = __reduce_max_sync(FULL, hi);
    bool e1 = cand && hi == mhi;
    unsigned mlo = __reduce_max_sync(FULL, e1 ? lo : 0u);
    bool e2 = e1 && lo == mlo;
    unsigned r = __reduce_min_sync(FULL, e2 ? (unsigned)row : 0xffffffffu);
    kout = ((unsigned long long)mhi << 32) | mlo;
    rout = (int)r;  // 0xffffffff -> -1
}

// Warp arg-max as above, returning the WINNING LANE (-1: no candidate); the
// winner knows its own key and row.  Common case: one redux on the high word
// of the key and a ballot; the exact low-word compare and the smallest-row
// rule run only when two candidates share the high word.
__device__ __forceinline__ int warp_argmax_lane(bool cand, unsigned long long key, int row) {
    const unsigned hi = cand ? (unsigned)(key >> 32) : 0u;
    const unsigned mhi = __reduce_max_sync(FULL, hi);
    const bool e1 = cand && hi == mhi;
    unsigned wm = __ballot_sync(FULL, e1);
    if (wm & (wm - 1)) {
        const unsigned mlo = __reduce_max_sync(FULL, e1 ? (unsigned)key : 0u);
        const bool e2 = e1 && (unsigned)key == mlo;
        const unsigned r = __reduce_min_sync(FULL, e2 ? (unsigned)row : 0xffffffffu);
        wm = __ballot_sync(FULL, e2 && (unsigned)row == r);
    }
    return wm ? __ffs(wm) - 1 : -1;
}

// 1/x for normal x whose reciprocal is normal, else 0 (the caller divides:
// LAPACK divides below sfmin).  MUFU.RCP64H seed + one cubic Newton step:
// error ~2^-66 before the final rounding, so the result is exact whenever
// 1/x is representable (the dyadic test families) and within 1 ulp otherwise
// (SURVEY Q6).  Cheap enough to run speculatively on every candidate, off the
// pivot-search critical path.
__device__ __forceinline__ double fast_rcp(double x) {
    const double ax = fabs(x);
    double r;
    asm("rcp.approx.ftz.f64 %0, %1;" : "=d"(r) : "d"(x));
    const double e = fma(-x, r, 1.0);
    r = fma(r, fma(e, e, e), r);
    return (ax >= DBL_MIN && ax <= 0x1p1021) ? r : 0.0;
}

// Pivot scaling as LAPACK dgetf2: multiply by the reciprocal when
// |pivot| >= sfmin, else divide (the tolerance absorbs the 1 ulp).
struct PivotScale {
    double pv, rcp;
    bool use_rcp;
    __device__ __forceinline__ explicit PivotScale(double p) : pv(p) {
        use_rcp = fabs(p) >= DBL_MIN;
        rcp = use_rcp ? __drcp_rn(p) : 0.0;
    }
    __device__ __forceinline__ double operator()(double v) const { return use_rcp ? v * rcp : v / pv; }
};

__device__ __forceinline__ int imin(int a, int b) { return a < b ? a : b; }
__device__ __forceinline__ int imax(int a, int b) { return a > b ? a : b; }

// ---------------------------------------------------------------- async staging
// cp.async (LDGSTS): global -> shared without registers, so a whole matrix
// or panel is in flight at once instead of one dependent load per iteration.
__device__ __forceinline__ void cp_async8(void *smem, const void *gmem) {
    unsigned s = (unsigned)__cvta_generic_to_shared(smem);
    asm volatile("cp.async.ca.shared.global [%0], [%1], 8;\n" ::"r"(s), "l"(gmem) : "memory");
}
__device__ __forceinline__ void cp_async16(void *smem, const void *gmem) {
    unsigned s = (unsigned)__cvta_generic_to_shared(smem);
    asm volatile("cp.async.cg.shared.global [%0], [%1], 16;\n" ::"r"(s), "l"(gmem) : "memory");
}
__device__ __forceinline__ void cp_async_commit() { asm volatile("cp.async.commit_group;\n" ::: "memory"); }
template <int N>
__device__ __forceinline__ void cp_async_wait() {
    asm volatile("cp.async.wait_group %0;\n" ::"n"(N) : "memory");
}

// Copy an m x n column-major block (leading dim ld) into shared memory with
// leading dim lds, issued by `nthr` threads starting at thread `t0`
// (cooperative).  Uses 16-byte copies when the block is one contiguous,
// 16-byte aligned range in both spaces, else 8-byte copies per element.
__device__ __forceinline__ void stage_block_async(double *s, int lds, const double *g, long ld, int m, int n,
                                                  int t, int nthr) {
    const int total = m * n;
    if (ld == m && lds == m) {
        const bool al = ((((uintptr_t)s) | ((uintptr_t)g)) & 15) == 0;
        if (al) {
            const int pairs = total >> 1;
            for (int e = t; e < pairs; e += nthr) cp_async16(s + 2 * e, g + 2 * e);
            if ((total & 1) && t == 0) cp_async8(s + total - 1, g + total - 1);
        } else {
            for (int e = t; e < total; e += nthr) cp_async8(s + e, g + e);
        }
    } else {
        // warps over columns, lanes over rows: no per-element integer division
        const int lane = t & 31, w0 = t >> 5, nw = nthr >> 5;
        for (int c = w0; c < n; c += nw) {
            const double *gc = g + (size_t)c * ld;
            double *sc = s + c * lds;
            for (int r = lane; r < m; r += 32) cp_async8(sc + r, gc + r);
        }
    }
}

// ---------------------------------------------------------------- launchers (host)
struct GetrfArgs {
    int batch, max_m, max_n;
    const int *m, *n;
    double *const *A;
    const int *ld;
    int *const *ipiv;
    int *info;
};

// zgetrf.cu: complex LU (interleaved re / im, ld in complex elements)
struct ZArgs {
    int batch, max_m, max_n;
    const int *m, *n;
    double *const *A;
    const int *ld;
    int *const *ipiv;
    int *info;
};
void launch_zgetrf(const ZArgs &a, int *counters, int *keys, int *sort_ws, cudaStream_t s);

// classify.cu
void launch_extend_add(int batch, int max_n2, const int *n2, const double *const *F22, const int *ld22,
                       const int *const *rel, const int *np, double *const *Fp, const int *ldp, int *info,
                       cudaStream_t s);
void launch_classify(const GetrfArgs &a, int *counters, int *bins, int keep_neg_info, cudaStream_t s);
void launch_max_dims(int batch, const int *m, const int *n, int *counters, cudaStream_t s);

// lu_small.cu
// optional second stream for the narrow classes (their kernels fill the wide
// classes' tails): fork recorded on s, joined back into s
struct SmallStreams {
    cudaStream_t s2;
    cudaEvent_t fork, join;
};
void launch_lu_small(const GetrfArgs &a, const int *counters, const int *bins, cudaStream_t s,
                     const SmallStreams *ss = nullptr);
// lu_mid.cu
void launch_lu_mid(const GetrfArgs &a, const int *counters, const int *bins, int bin, int max_elems,
                   cudaStream_t s);
// lu_large.cu
constexpr size_t SWAP_PLAN_BYTES = 1040;  // sizeof(SwapPlan), checked in lu_large.cu
constexpr int NB_OUTER_MAX = 128;          // widest outer block of the two-level grid tier
constexpr size_t OUTER_PLAN_BYTES = 2064;  // sizeof(OuterPlan), checked in lu_large.cu
// second part of the two-level grid tier (tuning parts = 2): its own counters
// block, list, tile offsets and stream
struct PartWork {
    int *counters;  // CNT_INTS ints
    int *list;      // batch ints
    int *tile_off;  // batch + 1 ints
    cudaStream_t side;
    cudaEvent_t fork, join;
};
void launch_lu_large(const GetrfArgs &a, int *counters, const int *bins, int *tile_off, void *plans, void *outer_plans,
                     cudaStream_t s, int *keys = nullptr, int *sort_ws = nullptr, PartWork *pw = nullptr);
void launch_lu_l1(const GetrfArgs &a, int *counters, const int *bins, int *keys, int *sort_ws, cudaStream_t s);

// gemm_vb.cu : DCWI gemm on pointer arrays (irr_gemm semantics)
struct GemmArgs {
    int ta, tb, max_m, max_n, max_k;
    const int *m, *n, *k;
    double alpha, beta;
    const double *const *A; int Ai, Aj; const int *lda;
    const double *const *B; int Bi, Bj; const int *ldb;
    double *const *C; int Ci, Cj; const int *ldc;
    int batch;
};
void launch_gemm_dcwi(const GemmArgs &g, int *counters, int *tile_off, cudaStream_t s);

// trsm_vb.cu
struct TrsmArgs {
    int side, uplo, trans, diag, max_m, max_n;
    const int *m, *n;
    double alpha;
    const double *const *T; int Ti, Tj; const int *ldt;
    double *const *B; int Bi, Bj; const int *ldb;
    int batch;
};
void run_trsm(const TrsmArgs &t, int *counters, int *tile_off, cudaStream_t s);

// laswp_vb.cu
void launch_laswp(int max_n, const int *n, double *const *A, int Ai, int Aj, const int *lda, int k1, int k2,
                  const int *kcount, int *const *ipiv, int batch, cudaStream_t s);

// partial.cu
void launch_partial_validate(int batch, int max_n1, int max_n2, const int *n1, const int *n2,
                             const int *ld11, const int *ld12, const int *ld21, const int *ld22,
                             double *const *F11, double *const *F12, const double *const *F21,
                             double *const *F22, int *const *ipiv, int *info, cudaStream_t s);

void launch_getrs_validate(int batch, int max_n, int max_nrhs, const int *n, const int *nrhs,
                           const double *const *A, const int *lda, int *const *ipiv, double *const *B,
                           const int *ldb, int *info, cudaStream_t s);

void launch_status_words(int batch, const int *m, const int *n, int *const *ipiv, const int *info, unsigned *words,
                         cudaStream_t s);

int num_sms();

// Raise a kernel's dynamic shared-memory limit to >= `bytes` on the CURRENT
// device (the attribute is per device).  Cached per (kernel, device) under a
// lock, so repeated launches cost a map lookup; never called on a kernel path.
cudaError_t smem_optin_fn(const void *func, size_t bytes);
template <class K>
inline cudaError_t smem_optin(K *kernel, size_t bytes) {
    return smem_optin_fn(reinterpret_cast<const void *>(kernel), bytes);
}
}  // namespace irr

#define IRR_CUDA_TRY(x)                                  \
    do {                                                 \
        cudaError_t e__ = (x);                           \
        if (e__ != cudaSuccess) return IRR_ERR_CUDA;     \
    } while (0)

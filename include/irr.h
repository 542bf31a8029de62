/*
 * irr.h -- C ABI of the B200-native irrLU library (libirr.so).
 *
 * Variable-size ("irregular") batched dense LU with partial pivoting and its
 * building blocks, after Abdelfattah et al., SC'22.  Citations "P:L<n>" are
 * lines of the paper text (/root/reference/PAPER.md at build time).
 *
 * CONVENTIONS (apply to every call)
 *  - All arrays and pointers are DEVICE memory unless marked (host).  int is
 *    32-bit.  Matrices are column-major FP64.  Pivot indices are
 *    1-based (LAPACK), local to each matrix.
 *  - Required dimensions (host scalars, e.g. max_m) describe the operation for
 *    the LARGEST matrix of the batch.  Local dimensions (device int
 *    arrays m[], n[], k[]) describe each matrix and are never modified
 *    (P:L129).  Pointer offsets (host scalars Xi, Xj) select the submatrix
 *    X[id] = Xarray[id] + Xj*ldx[id] + Xi of every matrix.
 *  - Dynamic Compute-Workload Inference, DCWI: every kernel
 *    infers the actual per-matrix work from required dims, local dims and
 *    offsets; a matrix with no remaining work does nothing.  There is no
 *    per-matrix host loop anywhere in the library.
 *  - Ownership: the caller owns ALL memory (matrices, pointer arrays, size
 *    arrays, ipiv, info, workspace).  The library never allocates on the hot
 *    path; its only state is a per-device property cache created on first use.
 *    The caller-provided workspace keeps the calls asynchronous.
 *  - Asynchrony: every call enqueues work on `stream` and returns without
 *    synchronising, except irr_getrf / irr_getrf_partial when a required
 *    dimension is passed as <= 0: then the library computes it with one device
 *    reduction and one device-to-host copy (documented synchronisation).
 *  - Return value: IRR_SUCCESS (0); -p if host argument p (1-based position in
 *    the C signature) is invalid; IRR_ERR_* (> 0) for a workspace that is too
 *    small, a launch failure or an unsupported device.  Per-matrix errors are
 *    reported in info[] (see irr_getrf).
 *  - Aliasing: matrices, ipiv arrays and workspace must not overlap.
 *  - Device: compiled for sm_100a only (B200); any other device gives
 *    IRR_ERR_DEVICE.
 */
#ifndef IRR_H
#define IRR_H

#include <stddef.h>

#ifdef __cplusplus
extern "C" {
#endif

/* Opaque CUDA stream handle (binary-compatible with cudaStream_t). NULL is the
 * legacy default stream. */
typedef struct CUstream_st *irr_stream_t;

typedef enum { IRR_NO_TRANS = 0, IRR_TRANS = 1 } irr_trans_t;
typedef enum { IRR_LEFT = 0, IRR_RIGHT = 1 } irr_side_t;
typedef enum { IRR_LOWER = 0, IRR_UPPER = 1 } irr_uplo_t;
typedef enum { IRR_NON_UNIT = 0, IRR_UNIT = 1 } irr_diag_t;

#define IRR_SUCCESS 0
#define IRR_ERR_CUDA 1        /* a CUDA launch or API call failed              */
#define IRR_ERR_WORKSPACE 2   /* work_bytes < the *_workspace_size() query     */
#define IRR_ERR_UNSUPPORTED 3 /* size or option outside what this build does   */
#define IRR_ERR_DEVICE 4      /* current device is not sm_100 (B200)           */

/* ------------------------------------------------------------------------
 * irr_getrf -- batched LU with partial pivoting on matrices of different
 * sizes: P_i L_i U_i = A_i for every i (§III-B; irrLU).
 *
 *  batch        (host) number of matrices, >= 0.
 *  max_m, max_n (host) required dims = max_i m[i], max_i n[i].
 *               Must be >= every m[i], n[i]; matrices exceeding them get
 *               info[i] = -1 / -2.  Pass <= 0 to have them computed (1 sync).
 *  m, n         local dims, int[batch].
 *  A            double*[batch]; A[i] points to an m[i] x n[i] column-major
 *               matrix with leading dimension ld[i].  Overwritten
 *               by L (unit lower, strictly below the diagonal) and U (upper,
 *               including the diagonal).
 *  ld           int[batch], ld[i] >= max(1, m[i]).
 *  ipiv         int*[batch]; ipiv[i] -> int[min(m[i], n[i])]: row k (1-based
 *               k+1) was interchanged with row ipiv[i][k] at step k.
 *  info         int[batch] output.  0: success.  k > 0: U(k,k) (1-based) is an
 *               exact zero; the factorization still completes (LAPACK).
 *               -1 / -2 / -3 / -4 / -5: bad m[i] / n[i] / A[i] / ld[i] /
 *               ipiv[i] (LAPACK argument positions); the matrix is skipped.
 *  work         device workspace of >= irr_getrf_workspace_size(batch, max_m,
 *               max_n) bytes, 256-byte aligned, caller-owned.
 *  stream       CUDA stream; the call is asynchronous on it.
 * Pivot search picks the largest |a_ik| with the smallest row index on ties
 * (BLAS idamax).  Results of matrix i depend only on (m[i], n[i], A[i]), not
 * on the rest of the batch.
 * ---------------------------------------------------------------------- */
size_t irr_getrf_workspace_size(int batch, int max_m, int max_n);
int irr_getrf(int batch, int max_m, int max_n, const int *m, const int *n, double *const *A,
              const int *ld, int *const *ipiv, int *info, void *work, size_t work_bytes,
              irr_stream_t stream);

/* ------------------------------------------------------------------------
 * irr_getrf_partial -- partial factorization of a batch of frontal matrices
 * F = [F11 F12; F21 F22] (multifrontal step, §III-A):
 *      P L U <- LU(F11)              pivoting restricted to F11's rows
 *      F12   <- U^-1 L^-1 P^T F12
 *      F22   <- F22 - F21 F12        (Schur complement; F21 is NOT modified)
 *  n1, n2       local dims, int[batch]: F11 n1 x n1, F12 n1 x n2, F21 n2 x n1,
 *               F22 n2 x n2.  max_n1 / max_n2 (host) their maxima (<= 0: computed).
 *  F11..F22     double*[batch] with leading dims ld11..ld22 (int[batch]); the
 *               four blocks may be parts of one nf x nf front (ld = nf).
 *  ipiv         int*[batch] -> int[n1[i]];  info int[batch] as for irr_getrf
 *               (bad n1 -> -1, n2 -> -2, ld11 -> -4, ld12 -> -6, ld21 -> -8,
 *               ld22 -> -10).  A zero pivot (info > 0) still runs the F12/F22
 *               updates with IEEE inf/NaN semantics.
 *  work         >= irr_getrf_partial_workspace_size(batch, max_n1, max_n2).
 * ---------------------------------------------------------------------- */
size_t irr_getrf_partial_workspace_size(int batch, int max_n1, int max_n2);
int irr_getrf_partial(int batch, int max_n1, int max_n2, const int *n1, const int *n2,
                      double *const *F11, const int *ld11, double *const *F12, const int *ld12,
                      const double *const *F21, const int *ld21, double *const *F22, const int *ld22,
                      int *const *ipiv, int *info, void *work, size_t work_bytes, irr_stream_t stream);

/* ------------------------------------------------------------------------
 * irr_getrf_partial_lapack -- the LAPACK-style variant of the partial front
 * factorization (the factors a solver keeps):
 *      P L U <- LU(F11)              pivoting restricted to F11's rows
 *      F12   <- U12 = L^-1 P^T F12   (interchanges + unit-lower solve)
 *      F21   <- L21 = F21 U^-1       (F21 IS overwritten)
 *      F22   <- F22 - L21 U12        (the same Schur complement as
 *                                     irr_getrf_partial in exact arithmetic)
 * Arguments, layouts, ownership, per-front info and host errors exactly as
 * irr_getrf_partial (F21 is writable here).  Built from the library's own
 * building blocks (irrLASWP, irrTRSM left-lower-unit and right-upper, irrGEMM).
 *  work         >= irr_getrf_partial_lapack_workspace_size(batch, ...).
 * ---------------------------------------------------------------------- */
size_t irr_getrf_partial_lapack_workspace_size(int batch, int max_n1, int max_n2);
int irr_getrf_partial_lapack(int batch, int max_n1, int max_n2, const int *n1, const int *n2,
                             double *const *F11, const int *ld11, double *const *F12, const int *ld12,
                             double *const *F21, const int *ld21, double *const *F22, const int *ld22,
                             int *const *ipiv, int *info, void *work, size_t work_bytes, irr_stream_t stream);

/* ------------------------------------------------------------------------
 * irr_zgetrf -- variable-size batched COMPLEX LU with partial pivoting
 * (the multifrontal solver's A is in C^{N x N},
 * P:L71 §III-A), LAPACK zgetrf semantics: P A = L U with the pivot of step
 * k the smallest row maximising |Re a_ik| + |Im a_ik| (izamax).
 *  A            double*[batch]: A_i -> m_i x n_i COMPLEX matrix, column-major,
 *               each element two doubles (re, im) as in C99 double _Complex /
 *               std::complex<double>; 16-byte aligned; ld[i] in complex
 *               elements (>= max(1, m_i)).  Overwritten by L (unit, strict
 *               lower) and U.
 *  m, n, ipiv, info, max_m, max_n, work, stream: exactly as irr_getrf
 *               (per-matrix info -1 / -2 / -3 / -4 / -5 for bad m / n / NULL
 *               A_i / ld / NULL ipiv_i; first exact zero pivot -> info = k).
 *  work         >= irr_zgetrf_workspace_size(batch, max_m, max_n).
 * ---------------------------------------------------------------------- */
size_t irr_zgetrf_workspace_size(int batch, int max_m, int max_n);
int irr_zgetrf(int batch, int max_m, int max_n, const int *m, const int *n, double *const *A, const int *ld,
               int *const *ipiv, int *info, void *work, size_t work_bytes, irr_stream_t stream);

/* ------------------------------------------------------------------------
 * irr_shard_lpt / irr_shard_lpt_work -- flop-balanced partition of a batch
 * over `parts` GPUs of one box (north_star: "fronts are
 * partitioned flop-balanced across the GPUs").  HOST arrays, host code, no
 * CUDA.  Longest-processing-time first: items by work descending (index
 * ascending on ties), each to the least-loaded part (lowest id on ties);
 * deterministic.  irr_shard_lpt weighs matrix i by FLOPS_DGETRF(m[i], n[i])
 * (reading Q1); irr_shard_lpt_work takes the weights (e.g. partial-front
 * flops, reading Q2).  owner[i] in [0, parts).  Returns 0 or -(position) of
 * a bad argument.
 * ---------------------------------------------------------------------- */
int irr_shard_lpt(int batch, const int *m, const int *n, int parts, int *owner);
int irr_shard_lpt_work(int batch, const double *work, int parts, int *owner);

/* ------------------------------------------------------------------------
 * irr_gemm -- irrGEMM (§IV-C) with the expanded interface:
 *      C_i <- alpha op(A_i) op(B_i) + beta C_i      (beta == 0: C not read)
 * Local dims: C_i is m[i] x n[i]; op(A_i) is m[i] x k[i]; op(B_i) is k[i] x n[i]
 * (so A_i is stored m x k, or k x m when ta == IRR_TRANS).  Offsets select
 * submatrices; DCWI clamps the required dims (max_m, max_n, max_k):
 *   m_eff = min(max_m, m_i - rowoff(op A), m_i - Ci)
 *   n_eff = min(max_n, n_i - coloff(op B), n_i - Cj)
 *   k_eff = min(max_k, k_i - coloff(op A), k_i - rowoff(op B))
 * where for op(A) = A^T the offsets (Ai, Aj) are compared against (k, m)
 * instead of (m, k).  A matrix with m_eff <= 0 or n_eff <= 0 does
 * nothing; k_eff <= 0 gives C <- beta C.
 *  work / work_bytes: optional (may be NULL/0).  With a workspace of
 *  irr_gemm_workspace_size(batch) bytes the tile schedule is built on the
 *  device (balanced); without one, a DCWI grid over the required dims is used.
 * ---------------------------------------------------------------------- */
size_t irr_gemm_workspace_size(int batch);
int irr_gemm(irr_trans_t ta, irr_trans_t tb, int max_m, int max_n, int max_k, const int *m, const int *n,
             const int *k, double alpha, const double *const *A, int Ai, int Aj, const int *lda,
             const double *const *B, int Bi, int Bj, const int *ldb, double beta, double *const *C, int Ci,
             int Cj, const int *ldc, int batch, void *work, size_t work_bytes, irr_stream_t stream);

/* ------------------------------------------------------------------------
 * irr_trsm -- irrTRSM (§IV-D): in-place triangular solve,
 *      side = LEFT : op(T_i) X = alpha B_i      (T_i is m[i] x m[i])
 *      side = RIGHT: X op(T_i) = alpha B_i      (T_i is n[i] x n[i])
 * B_i (m[i] x n[i]) is overwritten by X.  uplo / diag describe the stored T;
 * only that triangle is read (the diagonal is not read when diag = UNIT).
 * Recursive on the required dims, the off-diagonal blocks being
 * irrGEMM calls; DCWI clamps: left m_eff = min(max_m, m_i - Ti, m_i - Tj,
 * m_i - Bi), n_eff = min(max_n, n_i - Bj); right symmetrically on n.
 *  work: optional, as for irr_gemm (irr_trsm_workspace_size(batch)).
 * ---------------------------------------------------------------------- */
size_t irr_trsm_workspace_size(int batch);
int irr_trsm(irr_side_t side, irr_uplo_t uplo, irr_trans_t trans, irr_diag_t diag, int max_m, int max_n,
             const int *m, const int *n, double alpha, const double *const *T, int Ti, int Tj,
             const int *ldt, double *const *B, int Bi, int Bj, const int *ldb, int batch, void *work,
             size_t work_bytes, irr_stream_t stream);

/* ------------------------------------------------------------------------
 * irr_laswp -- irrLASWP (§IV-F): row interchanges
 *      for k = k1 .. k2-1:  swap rows k and ipiv[i][k]-1 of A_i
 * (rows relative to the offset Ai), applied to the columns
 * [Aj, Aj + min(max_n, n_i - Aj)) of A_i; k2 is clamped to kcount[i]
 * (the length of ipiv[i]).  n[i] is the local column count of A_i; rows must
 * exist (ipiv entries < lda rows are the caller's contract).  The composite
 * permutation is "rehearsed" on an index vector first and the rows are then
 * moved once each.
 * ---------------------------------------------------------------------- */
int irr_laswp(int max_n, const int *n, double *const *A, int Ai, int Aj, const int *lda, int k1, int k2,
              const int *kcount, int *const *ipiv, int batch, irr_stream_t stream);

/* ------------------------------------------------------------------------
 * irr_getrs -- batched solve with the factors of irr_getrf (SURVEY §8(f)
 * NEXT 1; the GETRS composition the paper benchmarks irrTRSM against, P:L96,
 * L215, and the solve step of P:L77-79):
 *      X_i <- A_i^-1 B_i = U_i^-1 L_i^-1 P_i^T B_i
 *  trans        IRR_NO_TRANS only (IRR_TRANS -> IRR_ERR_UNSUPPORTED).
 *  n, nrhs      int[batch]: A_i is n[i] x n[i] holding L\U and ipiv[i] as
 *               irr_getrf left them; B_i is n[i] x nrhs[i] (column-major,
 *               leading dimension ldb[i] >= max(1, n[i])), overwritten by X_i.
 *               max_n / max_nrhs (host) bound them (<= 0: computed, one sync).
 *  A, lda, ipiv, B, ldb   device pointer / int arrays as for irr_getrf.
 *  info         int[batch] (output): 0, or -(argument position) for a bad
 *               n (-5), nrhs (-6), NULL A_i (-7), lda (-8), NULL ipiv_i or a
 *               pivot ipiv_i[k] outside [k+1, n_i] (-9), NULL B_i (-10) or
 *               ldb (-11); those systems are skipped.  No
 *               singularity check (LAPACK dgetrs): a zero U_ii gives IEEE
 *               inf / NaN in X_i.
 *  work         >= irr_getrs_workspace_size(batch) bytes (caller-owned).
 * Host errors: -1 trans, -2 batch, -(position) for NULL arrays, as above.
 * Asynchronous on `stream` when max_n and max_nrhs are given.
 * ---------------------------------------------------------------------- */
size_t irr_getrs_workspace_size(int batch);
int irr_getrs(irr_trans_t trans, int batch, int max_n, int max_nrhs, const int *n, const int *nrhs,
              const double *const *A, const int *lda, int *const *ipiv, double *const *B, const int *ldb,
              int *info, void *work, size_t work_bytes, irr_stream_t stream);

/* ------------------------------------------------------------------------
 * irr_status_words -- the per-matrix completion record gathered across GPUs
 * (SURVEY §8(a) a6 / §8(e)): words[2 i] = info[i], words[2 i + 1] = 32-bit
 * FNV-1a hash (offset basis 2166136261, prime 16777619) of the bytes of
 * ipiv[i][0 .. min(m[i], n[i])) in little-endian order (0 entries: the basis;
 * matrices with info[i] < 0: 0).  All arrays device memory; asynchronous on
 * `stream`; returns 0 or IRR_ERR_CUDA.
 * ---------------------------------------------------------------------- */
int irr_status_words(int batch, const int *m, const int *n, int *const *ipiv, const int *info,
                     unsigned int *words, irr_stream_t stream);

/* ------------------------------------------------------------------------
 * irr_extend_add -- batched extend-add of child Schur complements into their
 * parent fronts.  PAPER.md L99 §III-A: "After these
 * operations are applied to front F_r, the Schur complement F_{r:22} is added
 * into the parent frontal matrix ... this requires a scatter operation";
 * L102: all fronts of one tree level are handled concurrently.  For child c:
 *     Fp_c[rel_c[i], rel_c[j]] += F22_c[i, j]     0 <= i, j < n2[c]
 *  batch        number of children (>= 0)                               (host)
 *  max_n2       >= every n2[c]; 0 => nothing to do                      (host)
 *  n2[batch]    order of each child's Schur complement
 *  F22[batch]   -> column-major n2 x n2 Schur complement (read only), ld22[c]
 *  rel[batch]   -> int[n2[c]]: 0-based row / column of the parent front that
 *               the child's row / column i maps to (distinct entries)
 *  np[batch]    order of the parent front of child c
 *  Fp[batch]    -> column-major np x np parent front of child c (several
 *               children may point at the same parent), ldp[c]
 *  info[batch]  0, or -(argument position) of the first bad per-child value:
 *               -3 n2 < 0 or > max_n2, -5 ld22 < max(1, n2), -6 a rel entry
 *               outside [0, np), -7 np < 0, -9 ldp < max(1, np), -4 / -8 NULL
 *               F22 / Fp with n2 > 0; such a child adds nothing.
 * The adds are atomic (FP64 reductions in L2): children sharing a parent may
 * be in one call; an entry hit by one child per call gets exactly
 * fl(Fp + F22) (bit-identical to a sequential sum), an entry hit by several
 * children of one call gets their sum in an unspecified order.  Call once per
 * sibling round (child 0s, then child 1s) for a result independent of
 * scheduling.  All arrays device memory, caller-owned; asynchronous on
 * `stream`.  Host errors: -1 batch, -2 max_n2, -(position) for NULL arrays.
 * ---------------------------------------------------------------------- */
int irr_extend_add(int batch, int max_n2, const int *n2, const double *const *F22, const int *ld22,
                   const int *const *rel, const int *np, double *const *Fp, const int *ldp, int *info,
                   irr_stream_t stream);

/* ------------------------------------------------------------------------
 * Tuning (tests and experiments; defaults are fixed by measurement and are
 * process-global, not thread-safe).  Keys: "nb" (tier-L panel width, 1..64),
 * "tier_s" (1 = enable the warp-per-matrix tier, 2 = also pack 4 / 2 matrices
 * per warp when m, n <= 8 / 16; default 2), "tier_m_max" (max padded
 * m*n of the shared-memory tier, 0 disables it), "l1" (1 = CTA-per-matrix
 * tier for m <= 256), "l1_ctas_per_sm" (1..3), "panel_rows" (max rows of a
 * grid-wide panel staged in shared memory), "trsm_nb" (TRSM recursion leaf),
 * "concurrent" (1 = S/M tiers on a forked stream), "dmma" (1 = grid-wide GEMMs
 * on the FP64 tensor core), "l1_dmma" (same inside L1), "panel_win" (1 =
 * grid-wide panels of <= 2048 rows by the windowed register panel, 0 = the
 * shared-memory / global-memory panels), "strip" (1 = grid-wide tier fuses
 * interchange + TRSM + trailing GEMM per 64-column strip; needs panel_win),
 * "phase_timing" (1 = per-phase cycle
 * counters in the workspace), "nb_outer" (outer block of the two-level grid
 * tier, 0 = one level), "l1_rows" (max rows of the CTA-per-matrix tier),
 * "xgemm_warps" (trailing GEMM core: 8 or 16 warps, 9 = 8 DMMA warps + a
 * producer warpgroup on an mbarrier ring; default 9), "xgemm_tma" (1 = the
 * warp-specialised core's L21 operand by TMA bulk copies; default 1),
 * "mid_dmma" (1 = tier M's trailing update on the FP64 tensor core; default
 * 0), "outer_cols", "parts", "part_grid", "defer", "getrs_fused",
 * "getrs_vec".  Unknown keys are ignored;
 * irr_get_tuning returns the current value (-1 for an unknown key).
 * ---------------------------------------------------------------------- */
void irr_set_tuning(const char *key, int value);
int irr_get_tuning(const char *key);
void irr_reset_tuning(void);

/* Number of kernels this library launched on the calling thread since the
 * last reset (host-side count, used by the benchmark's gpu_launches). */
long long irr_launch_count(int reset);

/* ------------------------------------------------------------------------
 * Per-kernel-class device timing (benchmark instrumentation).  While enabled
 * every kernel the library launches is bracketed by two CUDA events on the
 * stream it is launched on.  irr_profile_enable(n) creates a pool for n
 * launches (0 disables and frees it); irr_profile_collect waits for the
 * recorded events, writes the summed milliseconds and launch counts per class
 * (arrays of nclass entries) and clears the record; returns the number of
 * launches read, -1 on a CUDA error.  Class c is named by
 * irr_profile_class_name(c); irr_profile_num_classes() gives the count.
 * ---------------------------------------------------------------------- */
int irr_profile_enable(int max_launches);
int irr_profile_collect(double *ms, long long *launches, int nclass);
/* Per class, the length of the UNION of its launches' [start, end] intervals
 * (ms) since the last collect -- differs from irr_profile_collect's sum when
 * kernels of one class run concurrently on several streams.  Does not clear
 * the record; call it before irr_profile_collect.  Returns the number of
 * launches read, -1 on a CUDA error. */
int irr_profile_busy(double *busy_ms, int nclass);
int irr_profile_num_classes(void);
const char *irr_profile_class_name(int c);

const char *irr_version(void);

#ifdef __cplusplus
}
#endif
#endif /* IRR_H */

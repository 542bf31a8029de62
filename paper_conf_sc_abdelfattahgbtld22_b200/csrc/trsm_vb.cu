// trsm_vb.cu -- irrTRSM (§IV-D): in-place triangular solve on
// matrices of different sizes, recursive on the required dimensions.
//
// "The host CPU coordinates the solve based on the largest dimensions ... the
// DCWI layer figures out the correct dimensions": the host splits the
// triangular dimension in halves; the off-diagonal blocks are irrGEMM calls
// (gemm_vb.cu) and the leaves are solved by trsm_leaf_kernel.  Unlike
// MAGMA-2.6.1 there is no explicit inverse of diagonal blocks and no
// out-of-place workspace copy: leaves use plain substitution with
// true division, in place.
#include "gemm_core.cuh"
#include "sched.cuh"

namespace irr {

void launch_gemm_masked(const GemmArgs &g, const int *mask, int *counters, int *tile_off, cudaStream_t s,
                        SlotList sl);

constexpr int TL = 32;        // leaf size (triangular dimension)
constexpr int TR_RHS = 128;   // right-hand sides per CTA
constexpr int TR_NT = 128;

struct LeafArgs {
    TrsmArgs t;
    const int *mask;
    int off;     // offset of this leaf along the triangular dimension
    int kt;      // required leaf size (<= TL)
    double alpha;
    int s_lower; // the solved system S x = b is lower triangular (forward)
    int tr;      // S(r, c) = T(c, r) when set, else T(r, c)
    int rhs_chunks;
};

// DCWI of one leaf for matrix i: effective triangle size and RHS count
__device__ __forceinline__ void leaf_dims(const LeafArgs &L, int i, int &kt, int &nrhs) {
    const TrsmArgs &t = L.t;
    kt = 0;
    nrhs = 0;
    if (L.mask && L.mask[i] < 0) return;
    const bool left = t.side == IRR_LEFT;
    const int mi = t.m[i], ni = t.n[i];
    const int tri = left ? mi : ni;  // local size of T
    kt = imin(L.kt, imin(tri - (t.Ti + L.off), tri - (t.Tj + L.off)));
    if (left) {
        kt = imin(kt, mi - (t.Bi + L.off));
        nrhs = imin(t.max_n, ni - t.Bj);
    } else {
        kt = imin(kt, ni - (t.Bj + L.off));
        nrhs = imin(t.max_m, mi - t.Bi);
    }
}

struct LeafUnits {
    LeafArgs L;
    __device__ int units(int i) const {
        int kt, nrhs;
        leaf_dims(L, i, kt, nrhs);
        return (kt > 0 && nrhs > 0) ? (nrhs + TR_RHS - 1) / TR_RHS : 0;
    }
};

// one (matrix, RHS chunk) leaf solve by the whole CTA
__device__ __forceinline__ void leaf_item(const LeafArgs &L, int i, int q, double (*S)[TL + 1],
                                          double (*buf)[TR_RHS + 1]) {
    const TrsmArgs &t = L.t;
    const int tid = threadIdx.x;
    const bool left = t.side == IRR_LEFT;
    int kt, nrhs;
    leaf_dims(L, i, kt, nrhs);
    const int toff_r = t.Ti + L.off, toff_c = t.Tj + L.off;
    {
        if (kt <= 0) return;
        const int r0 = q * TR_RHS;
        if (r0 >= nrhs) return;
        const int W = imin(TR_RHS, nrhs - r0);
        const long ldt = t.ldt[i], ldb = t.ldb[i];
        const double *T = t.T[i];
        double *B = t.B[i];
        // ---- S = the solved triangle (dense, zeros outside, unit diag)
        for (int e = tid; e < kt * kt; e += TR_NT) {
            const int r = e % kt, c = e / kt;
            const bool in = L.s_lower ? (r >= c) : (r <= c);
            double v = 0.0;
            if (r == c && t.diag == IRR_UNIT) v = 1.0;
            else if (in) {
                const int x = L.tr ? c : r, y = L.tr ? r : c;
                v = T[toff_r + x + (size_t)(toff_c + y) * ldt];
            }
            S[r][c] = v;
        }
        // ---- right-hand sides: left -> columns of B, right -> rows of B
        if (left) {
            for (int e = tid; e < kt * W; e += TR_NT) {
                const int r = e % kt, c = e / kt;
                buf[r][c] = B[t.Bi + L.off + r + (size_t)(t.Bj + r0 + c) * ldb];
            }
        } else {
            for (int e = tid; e < kt * W; e += TR_NT) {
                const int c = e % W, r = e / W;
                buf[r][c] = B[t.Bi + r0 + c + (size_t)(t.Bj + L.off + r) * ldb];
            }
        }
        __syncthreads();
        if (tid < W) {
            double x[TL];
#pragma unroll
            for (int r = 0; r < TL; ++r) x[r] = (r < kt) ? L.alpha * buf[r][tid] : 0.0;
            if (L.s_lower) {
#pragma unroll
                for (int sidx = 0; sidx < TL; ++sidx) {
                    if (sidx < kt) {
                        x[sidx] = x[sidx] / S[sidx][sidx];
#pragma unroll
                        for (int r = sidx + 1; r < TL; ++r)
                            if (r < kt) x[r] = fma(-S[r][sidx], x[sidx], x[r]);
                    }
                }
            } else {
#pragma unroll
                for (int sidx = TL - 1; sidx >= 0; --sidx) {
                    if (sidx < kt) {
                        x[sidx] = x[sidx] / S[sidx][sidx];
#pragma unroll
                        for (int r = 0; r < sidx; ++r) x[r] = fma(-S[r][sidx], x[sidx], x[r]);
                    }
                }
            }
#pragma unroll
            for (int r = 0; r < TL; ++r)
                if (r < kt) buf[r][tid] = x[r];
        }
        __syncthreads();
        if (left) {
            for (int e = tid; e < kt * W; e += TR_NT) {
                const int r = e % kt, c = e / kt;
                B[t.Bi + L.off + r + (size_t)(t.Bj + r0 + c) * ldb] = buf[r][c];
            }
        } else {
            for (int e = tid; e < kt * W; e += TR_NT) {
                const int c = e % W, r = e / W;
                B[t.Bi + r0 + c + (size_t)(t.Bj + L.off + r) * ldb] = buf[r][c];
            }
        }
        __syncthreads();
    }
}

// DCWI grid over (batch x RHS chunks of the required dims) (no workspace)
__global__ void __launch_bounds__(TR_NT) trsm_leaf_kernel(LeafArgs L) {
    __shared__ double S[TL][TL + 1];
    __shared__ double buf[TL][TR_RHS + 1];
    const long long total = (long long)L.t.batch * L.rhs_chunks;
    for (long long w = blockIdx.x; w < total; w += gridDim.x) {
        const int i = (int)(w / L.rhs_chunks), q = (int)(w - (long long)i * L.rhs_chunks);
        leaf_item(L, i, q, S, buf);
    }
}

// device-scheduled: only (matrix, chunk) units that exist, on the active slots
__global__ void __launch_bounds__(TR_NT) trsm_leaf_walk_kernel(LeafArgs L, SlotList sl, const int *off) {
    __shared__ double S[TL][TL + 1];
    __shared__ double buf[TL][TR_RHS + 1];
    walk_units(sl, L.t.batch, off, [&](int i, int q) { leaf_item(L, i, q, S, buf); });
}

namespace {

struct TrsmRec {
    TrsmArgs t;
    const int *mask;
    int *counters, *tile_off;
    int *sort_ws;  // size-sorted slots by the triangular dimension (nullptr: none)
    cudaStream_t s;
    int leaf;
    int m_lower;  // op(T) is lower triangular

    void leaf_solve(int off, int kt, double alpha) {
        LeafArgs L;
        L.t = t; L.mask = mask; L.off = off; L.kt = kt; L.alpha = alpha;
        const bool left = t.side == IRR_LEFT;
        // left: S = op(T); right: S = op(T)^T
        L.s_lower = left ? m_lower : !m_lower;
        // S(r,c) = op(T)(r,c) [left] or op(T)(c,r) [right]; op(T)(r,c) = T(c,r) iff trans
        L.tr = left ? (t.trans == IRR_TRANS) : (t.trans != IRR_TRANS);
        const int nrhs_max = left ? t.max_n : t.max_m;
        L.rhs_chunks = (nrhs_max + TR_RHS - 1) / TR_RHS;
        if (tile_off) {
            const SlotList sl = slots(off);
            {
                KScope k(K_GEMM_SCAN, s);
                scan_units_kernel<LeafUnits><<<1, 1024, 0, s>>>(LeafUnits{L}, sl, t.batch, tile_off);
            }
            KScope k(K_TRSM_LEAF, s);
            trsm_leaf_walk_kernel<<<num_sms() * 8, TR_NT, 0, s>>>(L, sl, tile_off);
            return;
        }
        long long total = (long long)t.batch * L.rhs_chunks;
        int grid = num_sms() * 8;
        if (total < grid) grid = (int)total;
        if (grid < 1) return;
        KScope k(K_TRSM_LEAF, s);
        trsm_leaf_kernel<<<grid, TR_NT, 0, s>>>(L);
    }

    // matrices whose triangular dimension exceeds `thr` (all when unsorted)
    SlotList slots(int thr) const { return sort_ws ? sorted_slots(sort_ws, t.batch, thr) : all_slots(); }

    // op(T) block with rows [R, R+nr) and columns [C, C+nc) as a GEMM operand
    void opT_operand(int R, int C, int &trans, int &oi, int &oj) const {
        if (t.trans == IRR_TRANS) { trans = 1; oi = t.Ti + C; oj = t.Tj + R; }
        else { trans = 0; oi = t.Ti + R; oj = t.Tj + C; }
    }

    // B_target <- beta * B_target - X * opT-block  or  - opT-block * X
    void update(int off_x, int nx, int off_c, int nc, double beta) {
        GemmArgs g{};
        g.batch = t.batch;
        g.alpha = -1.0;
        g.beta = beta;
        const bool left = t.side == IRR_LEFT;
        if (left) {
            // C = B rows [off_c, +nc) (all columns), op(A) = op(T)[off_c.., off_x..], B = X rows [off_x, +nx)
            int tr, oi, oj;
            opT_operand(off_c, off_x, tr, oi, oj);
            g.ta = tr; g.tb = 0;
            g.max_m = nc; g.max_n = t.max_n; g.max_k = nx;
            g.m = t.m; g.n = t.n; g.k = t.m;
            g.A = t.T; g.Ai = oi; g.Aj = oj; g.lda = t.ldt;
            g.B = (const double *const *)t.B; g.Bi = t.Bi + off_x; g.Bj = t.Bj; g.ldb = t.ldb;
            g.C = t.B; g.Ci = t.Bi + off_c; g.Cj = t.Bj; g.ldc = t.ldb;
        } else {
            // C = B cols [off_c, +nc), op(A) = X = B cols [off_x, +nx), op(B) = op(T)[off_x.., off_c..]
            int tr, oi, oj;
            opT_operand(off_x, off_c, tr, oi, oj);
            g.ta = 0; g.tb = tr;
            g.max_m = t.max_m; g.max_n = nc; g.max_k = nx;
            g.m = t.m; g.n = t.n; g.k = t.n;
            g.A = (const double *const *)t.B; g.Ai = t.Bi; g.Aj = t.Bj + off_x; g.lda = t.ldb;
            g.B = t.T; g.Bi = oi; g.Bj = oj; g.ldb = t.ldt;
            g.C = t.B; g.Ci = t.Bi; g.Cj = t.Bj + off_c; g.ldc = t.ldb;
        }
        launch_gemm_masked(g, mask, counters, tile_off, s, slots(off_x < off_c ? off_x : off_c));
    }

    void solve(int off, int K, double alpha) {
        if (K <= 0) return;
        if (K <= leaf) { leaf_solve(off, K, alpha); return; }
        int K1 = ((K / 2 + leaf - 1) / leaf) * leaf;
        if (K1 >= K) K1 = K - leaf;
        const int K2 = K - K1;
        const bool left = t.side == IRR_LEFT;
        // left:  solve order follows op(T): lower -> top first
        // right: X op(T) = B: op(T) upper -> first block first
        const bool first_block_first = left ? m_lower : !m_lower;
        if (first_block_first) {
            solve(off, K1, alpha);
            update(off, K1, off + K1, K2, alpha);
            solve(off + K1, K2, 1.0);
        } else {
            solve(off + K1, K2, alpha);
            update(off + K1, K2, off, K1, alpha);
            solve(off, K1, 1.0);
        }
    }
};

}  // namespace

// sort_ws: nullptr, or a size sort of the batch by the triangular dimension
// (launch_size_sort on t.m for LEFT, t.n for RIGHT) that TRSM levels use to
// visit only the matrices still active at their offset.
void run_trsm_masked(const TrsmArgs &t, const int *mask, int *counters, int *tile_off, cudaStream_t s,
                     int *sort_ws) {
    if (t.batch <= 0 || t.max_m <= 0 || t.max_n <= 0) return;
    TrsmRec R;
    R.t = t; R.mask = mask; R.counters = counters; R.tile_off = tile_off; R.s = s;
    R.sort_ws = tile_off ? sort_ws : nullptr;
    int leaf = tuning().trsm_nb;
    if (leaf < 1 || leaf > TL) leaf = TL;
    R.leaf = leaf;
    R.m_lower = (t.uplo == IRR_LOWER) != (t.trans == IRR_TRANS);
    const int K = t.side == IRR_LEFT ? t.max_m : t.max_n;
    R.solve(0, K, t.alpha);
}

void run_trsm(const TrsmArgs &t, int *counters, int *tile_off, cudaStream_t s) {
    run_trsm_masked(t, nullptr, counters, tile_off, s, nullptr);
}

}  // namespace irr

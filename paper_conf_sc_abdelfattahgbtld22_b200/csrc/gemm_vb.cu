// gemm_vb.cu -- irrGEMM with the expanded interface (§IV-A) and
// DCWI (§IV-B): C_i <- alpha op(A_i) op(B_i) + beta C_i on
// submatrices selected by scalar offsets, with per-matrix effective sizes
// inferred on the device.
#include "gemm_big.cuh"
#include "sched.cuh"

namespace irr {

struct DcwiGemmProb {
    GemmArgs g;
    const int *mask;  // optional: skip matrices with mask[i] < 0 (bad arguments)
    SlotList sl;      // slot -> matrix (identity, or a size-sorted prefix)
    __device__ bool get(int slot, GemmDesc &d) const {
        const int i = sl.matrix(slot);
        d.m = 0; d.n = 0; d.k = 0;
        if (mask && mask[i] < 0) return false;
        const int mi = g.m[i], ni = g.n[i], ki = g.k[i];
        // offsets of op(A) / op(B) in (rows, cols) of the op'ed operand: for
        // op(A) = A^T the stored (Ai, Aj) are compared against (k, m)
        const int a_m_off = g.ta ? g.Aj : g.Ai, a_k_off = g.ta ? g.Ai : g.Aj;
        const int b_k_off = g.tb ? g.Bj : g.Bi, b_n_off = g.tb ? g.Bi : g.Bj;
        int me = imin(g.max_m, imin(mi - a_m_off, mi - g.Ci));
        int ne = imin(g.max_n, imin(ni - b_n_off, ni - g.Cj));
        int ke = imin(g.max_k, imin(ki - a_k_off, ki - b_k_off));
        if (me <= 0 || ne <= 0) return false;
        if (ke < 0) ke = 0;
        d.m = me; d.n = ne; d.k = ke;
        d.ta = g.ta; d.tb = g.tb;
        d.alpha = g.alpha; d.beta = g.beta;
        const long ldc = g.ldc[i];
        d.C = g.C[i] + g.Ci + (size_t)g.Cj * ldc; d.ldc = ldc;
        if (ke > 0) {
            const long lda = g.lda[i], ldb = g.ldb[i];
            d.A = g.A[i] + g.Ai + (size_t)g.Aj * lda; d.lda = lda;
            d.B = g.B[i] + g.Bi + (size_t)g.Bj * ldb; d.ldb = ldb;
        } else {
            d.A = nullptr; d.B = nullptr; d.lda = 1; d.ldb = 1;
        }
        return true;
    }
};

void launch_gemm_masked(const GemmArgs &g, const int *mask, int *counters, int *tile_off, cudaStream_t s,
                        SlotList sl) {
    if (g.batch <= 0 || g.max_m <= 0 || g.max_n <= 0) return;
    const int sms = num_sms();
    if (tile_off) {
        DcwiGemmProb P{g, mask, sl};
        const int cnt = sl.prefix ? -1 : g.batch;
        const int *cnt_ptr = sl.prefix ? sl.prefix + sl.bucket0 : nullptr;
        // long-K products on the 128 x 128 DMMA core first, the rest on the
        // 64 x 64 core; both passes reuse tile_off (stream-ordered)
        const bool big = tuning().gemm_big && g.max_m >= 96 && g.max_n >= 96 && g.max_k >= 48;
        if (big) {
            using BP = SizeFilter<DcwiGemmProb>;
            BP Pb{P, 1};
            {
                KScope k(K_GEMM_SCAN, s);
                xgemm_scan_kernel<BP><<<1, 1024, 0, s>>>(Pb, cnt, cnt_ptr, tile_off);
            }
            KScope k(K_GEMM_DCWI, s);
            launch_xgemm(Pb, g.ta, g.tb, cnt, cnt_ptr, tile_off, s);
        }
        using SP = SizeFilter<DcwiGemmProb>;
        SP Ps{P, 0};
        if (!big) Ps.want_big = -1;  // no filtering
        {
            KScope k(K_GEMM_SCAN, s);
            gemm_scan_kernel<SP><<<1, 1024, 0, s>>>(Ps, cnt, cnt_ptr, tile_off);
        }
        KScope k(K_GEMM_DCWI, s);
        if (tuning().dmma) {
            gemm_smem_optin(gemm_sched_kernel<SP, true>);
            gemm_sched_kernel<SP, true><<<sms * 3, G_NT, GEMM_SMEM, s>>>(Ps, cnt, cnt_ptr, tile_off);
        } else {
            gemm_smem_optin(gemm_sched_kernel<SP, false>);
            gemm_sched_kernel<SP, false><<<sms * 3, G_NT, GEMM_SMEM, s>>>(Ps, cnt, cnt_ptr, tile_off);
        }
    } else {
        DcwiGemmProb P{g, mask, all_slots()};
        const int tm = (g.max_m + GBM - 1) / GBM, tn = (g.max_n + GBN - 1) / GBN;
        long long total = (long long)tm * tn * g.batch;
        int grid = sms * 4;
        if (total < grid) grid = (int)total;
        KScope k(K_GEMM_DCWI, s);
        if (tuning().dmma) {
            gemm_smem_optin(gemm_grid_kernel<DcwiGemmProb, true>);
            gemm_grid_kernel<DcwiGemmProb, true><<<grid, G_NT, GEMM_SMEM, s>>>(P, g.batch, tm, tn);
        } else {
            gemm_smem_optin(gemm_grid_kernel<DcwiGemmProb, false>);
            gemm_grid_kernel<DcwiGemmProb, false><<<grid, G_NT, GEMM_SMEM, s>>>(P, g.batch, tm, tn);
        }
    }
    (void)counters;
}

void launch_gemm_dcwi(const GemmArgs &g, int *counters, int *tile_off, cudaStream_t s) {
    launch_gemm_masked(g, nullptr, counters, tile_off, s, all_slots());
}

}  // namespace irr

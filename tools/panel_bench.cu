// panel_bench.cu -- cycles per column of the CTA panel factorizations in
// isolation (one CTA, panel already in shared memory).
//   nvcc -gencode arch=compute_100a,code=sm_100a -O3 -I include -I paper_conf_sc_abdelfattahgbtld22_b200/csrc \
//        -o tools/pb tools/panel_bench.cu && tools/pb
#include <cstdio>
#include "panel.cuh"

using namespace irr;

template <int NT, int RPT, int NBP>
__global__ void k_regs(const double *src, int rows, int ib, long long *cyc, int reps) {
    extern __shared__ double P[];
    __shared__ __align__(16) PanelRegScratch<NT / 32, NBP> prs;
    __shared__ int piv[64];
    const int ldp = rows | 1;
    long long tot = 0;
#ifdef IRR_PANEL_TIMING
    if (threadIdx.x < 8) s_ptime[threadIdx.x] = 0;
#endif
    for (int rep = 0; rep < reps; ++rep) {
        for (int c = 0; c < ib; ++c)
            for (int r = threadIdx.x; r < rows; r += NT) P[r + c * ldp] = src[r + c * rows];
        __syncthreads();
        long long t0 = clock64();
        panel_regs<NT, RPT, NBP>(P, ldp, rows, ib, piv, prs);
        long long t1 = clock64();
        tot += t1 - t0;
        __syncthreads();
    }
    if (threadIdx.x == 0) cyc[0] = tot / reps;
#ifdef IRR_PANEL_TIMING
    if (threadIdx.x < 8) g_ptime[threadIdx.x] = s_ptime[threadIdx.x];
#endif
}

template <int NT>
__global__ void k_getf2(const double *src, int rows, int ib, long long *cyc, int reps) {
    extern __shared__ double P[];
    __shared__ PanelScratch sc;
    __shared__ int piv[64];
    const int ldp = rows | 1;
    long long tot = 0;
    for (int rep = 0; rep < reps; ++rep) {
        for (int c = 0; c < ib; ++c)
            for (int r = threadIdx.x; r < rows; r += NT) P[r + c * ldp] = src[r + c * rows];
        __syncthreads();
        long long t0 = clock64();
        panel_getf2<NT>(P, ldp, 0, rows, 0, ib, 0, ib, piv, sc);
        long long t1 = clock64();
        tot += t1 - t0;
        __syncthreads();
    }
    if (threadIdx.x == 0) cyc[0] = tot / reps;
}

template <int NT, int RPT, int NBP>
void run_regs(const double *d, int rows, int ib, long long *dc, const char *name) {
    size_t smem = (size_t)(rows | 1) * ib * 8;
    cudaFuncSetAttribute(k_regs<NT, RPT, NBP>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
    cudaMemset(dc, 0, 8);
    k_regs<NT, RPT, NBP><<<1, NT, smem>>>(d, rows, ib, dc, 20);
    long long hc;
    cudaMemcpy(&hc, dc, 8, cudaMemcpyDeviceToHost);
    printf("%-28s %4dx%-3d: %.0f cycles/column\n", name, rows, ib, hc / (double)ib);
#ifdef IRR_PANEL_TIMING
    unsigned long long pt[8];
    cudaMemcpyFromSymbol(pt, g_ptime, sizeof(pt));
    const char *nm[6] = {"cand+warp_argmax+ballot", "publish", "barrier", "final argmax", "swap/U/pos/rcp", "update"};
    for (int k = 0; k < 6; ++k) printf("   %-24s %.0f cycles/column\n", nm[k], pt[k] / (20.0 * ib));
#endif
}

int main() {
    const int rows = 256, ib = 32;
    double *h = new double[1024 * 64];
    unsigned s = 12345;
    for (int i = 0; i < 1024 * 64; ++i) { s = s * 1664525u + 1013904223u; h[i] = (s >> 8) * (1.0 / 16777216.0) - 0.5; }
    double *d; long long *dc;
    cudaMalloc(&d, 1024 * 64 * 8); cudaMalloc(&dc, 8);
    cudaMemcpy(d, h, 1024 * 64 * 8, cudaMemcpyHostToDevice);
    run_regs<128, 2, 32>(d, 256, 32, dc, "regs<128,2,32>");
    run_regs<256, 1, 32>(d, 256, 32, dc, "regs<256,1,32>");
    run_regs<64, 2, 32>(d, 128, 32, dc, "regs<64,2,32> (128 rows)");
    run_regs<128, 1, 32>(d, 128, 32, dc, "regs<128,1,32> (128 rows)");
    run_regs<128, 2, 16>(d, 256, 16, dc, "regs<128,2,16>");
    run_regs<32, 2, 32>(d, 64, 32, dc, "regs<32,2,32> (64 rows)");
    printf("%s\n", cudaGetErrorString(cudaDeviceSynchronize()));
    return 0;
}

// panel_bench.cu -- cycles per column of the CTA panel factorizations in
// isolation (one CTA, panel already in shared memory).
//   nvcc -gencode arch=compute_100a,code=sm_100a -O3 -I include -I paper_conf_sc_abdelfattahgbtld22_b200/csrc \
//        -o tools/pb tools/panel_bench.cu && tools/pb
#include <cstdio>
#define IRR_PANEL_TIMING
#include "panel.cuh"

using namespace irr;

template <int NT, int RPT, int NBP>
__global__ void k_regs(const double *src, int rows, int ib, long long *cyc, int reps) {
    extern __shared__ double P[];
    __shared__ __align__(16) PanelRegScratch<NT / 32, NBP> prs;
    __shared__ int piv[64];
    const int ldp = rows | 1;
    long long tot = 0;
    if (threadIdx.x < 8) s_ptime[threadIdx.x] = 0;
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
    if (threadIdx.x < 8) g_ptime[threadIdx.x] = s_ptime[threadIdx.x];
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

int main() {
    const int rows = 256, ib = 32;
    double *h = new double[rows * ib];
    unsigned s = 12345;
    for (int i = 0; i < rows * ib; ++i) { s = s * 1664525u + 1013904223u; h[i] = (s >> 8) * (1.0 / 16777216.0) - 0.5; }
    double *d; long long *dc, hc;
    cudaMalloc(&d, rows * ib * 8); cudaMalloc(&dc, 8);
    cudaMemcpy(d, h, rows * ib * 8, cudaMemcpyHostToDevice);
    size_t smem = (size_t)(rows | 1) * ib * 8;
    cudaFuncSetAttribute(k_regs<128, 2, 32>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
    cudaFuncSetAttribute(k_getf2<128>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
    k_regs<128, 2, 32><<<1, 128, smem>>>(d, rows, ib, dc, 20);
    cudaMemcpy(&hc, dc, 8, cudaMemcpyDeviceToHost);
    printf("panel_regs<128,2,32>  256x32: %lld cycles, %.0f per column\n", hc, hc / 32.0);
    unsigned long long pt[8];
    cudaMemcpyFromSymbol(pt, g_ptime, sizeof(pt));
    const char *nm[6] = {"cand+warp_argmax+ballot", "publish", "barrier", "final argmax+u", "swap/U/pos/rcp", "update"};
    for (int k = 0; k < 6; ++k) printf("   %-24s %.0f cycles/column\n", nm[k], pt[k] / (20.0 * 32));
    k_getf2<128><<<1, 128, smem>>>(d, rows, ib, dc, 20);
    cudaMemcpy(&hc, dc, 8, cudaMemcpyDeviceToHost);
    printf("panel_getf2<128>      256x32: %lld cycles, %.0f per column\n", hc, hc / 32.0);
    printf("%s\n", cudaGetErrorString(cudaDeviceSynchronize()));
    return 0;
}

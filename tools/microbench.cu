// microbench.cu -- dependent-chain latencies of the operations on the panel's
// critical path (DFMA, REDUX, SHFL, LDS, BAR, DDIV/RCP), in SM cycles.
//   nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o /tmp/mb tools/microbench.cu && /tmp/mb
#include <cstdio>
#include <cuda_runtime.h>

#define N 2048

__global__ void k_dfma(double *out, long long *cyc, double a, double b) {
    double x = threadIdx.x;
    long long t0 = clock64();
#pragma unroll 16
    for (int i = 0; i < N; ++i) x = fma(x, a, b);
    long long t1 = clock64();
    out[threadIdx.x] = x;
    if (threadIdx.x == 0) cyc[0] = t1 - t0;
}

__global__ void k_redux(unsigned *out, long long *cyc) {
    unsigned x = threadIdx.x;
    long long t0 = clock64();
#pragma unroll 16
    for (int i = 0; i < N; ++i) x = __reduce_max_sync(0xffffffffu, x + threadIdx.x);
    long long t1 = clock64();
    out[threadIdx.x] = x;
    if (threadIdx.x == 0) cyc[0] = t1 - t0;
}

__global__ void k_shfl(double *out, long long *cyc) {
    double x = threadIdx.x;
    long long t0 = clock64();
#pragma unroll 16
    for (int i = 0; i < N; ++i) x = __shfl_sync(0xffffffffu, x, (threadIdx.x + 1) & 31) + 1.0;
    long long t1 = clock64();
    out[threadIdx.x] = x;
    if (threadIdx.x == 0) cyc[0] = t1 - t0;
}

__global__ void k_lds(int *out, long long *cyc) {
    __shared__ int s[1024];
    for (int i = threadIdx.x; i < 1024; i += blockDim.x) s[i] = (i + 1) & 1023;
    __syncthreads();
    int p = threadIdx.x;
    long long t0 = clock64();
#pragma unroll 16
    for (int i = 0; i < N; ++i) p = s[p];
    long long t1 = clock64();
    out[threadIdx.x] = p;
    if (threadIdx.x == 0) cyc[0] = t1 - t0;
}

__global__ void k_bar(int *out, long long *cyc) {
    __shared__ volatile int s[1024];
    int x = 0;
    long long t0 = clock64();
    for (int i = 0; i < N; ++i) {
        s[threadIdx.x] = i;
        __syncthreads();
        x += s[(threadIdx.x + 32) % blockDim.x];
    }
    long long t1 = clock64();
    out[threadIdx.x] = x;
    if (threadIdx.x == 0) cyc[0] = t1 - t0;
}

__global__ void k_rcp(double *out, long long *cyc, double a) {
    double x = a + threadIdx.x;
    long long t0 = clock64();
#pragma unroll 4
    for (int i = 0; i < N; ++i) x = 1.0 / x + 1.5;
    long long t1 = clock64();
    out[threadIdx.x] = x;
    if (threadIdx.x == 0) cyc[0] = t1 - t0;
}

__global__ void k_dfma_tput(double *out, long long *cyc, double a, double b) {
    double x[8];
    for (int j = 0; j < 8; ++j) x[j] = threadIdx.x + j;
    long long t0 = clock64();
    for (int i = 0; i < N; ++i) {
#pragma unroll
        for (int j = 0; j < 8; ++j) x[j] = fma(x[j], a, b);
    }
    long long t1 = clock64();
    double s = 0;
    for (int j = 0; j < 8; ++j) s += x[j];
    out[blockIdx.x * blockDim.x + threadIdx.x] = s;
    if (threadIdx.x == 0 && blockIdx.x == 0) cyc[0] = t1 - t0;
}

int main1() {
    double *dd; unsigned *du; int *di; long long *dc; long long hc;
    cudaMalloc(&dd, 1 << 20); cudaMalloc(&du, 1 << 20); cudaMalloc(&di, 1 << 20); cudaMalloc(&dc, 64);
    k_dfma<<<1, 32>>>(dd, dc, 1.0000001, 1e-9); cudaMemcpy(&hc, dc, 8, cudaMemcpyDeviceToHost);
    printf("DFMA dependent latency        %.1f cycles\n", (double)hc / N);
    k_redux<<<1, 32>>>(du, dc); cudaMemcpy(&hc, dc, 8, cudaMemcpyDeviceToHost);
    printf("REDUX.MAX (+IADD) latency     %.1f cycles\n", (double)hc / N);
    k_shfl<<<1, 32>>>(dd, dc); cudaMemcpy(&hc, dc, 8, cudaMemcpyDeviceToHost);
    printf("SHFL.f64x2 (+DADD) latency    %.1f cycles\n", (double)hc / N);
    k_lds<<<1, 32>>>(di, dc); cudaMemcpy(&hc, dc, 8, cudaMemcpyDeviceToHost);
    printf("LDS pointer chase             %.1f cycles\n", (double)hc / N);
    for (int nt : {32, 128, 256, 512}) {
        k_bar<<<1, nt>>>(di, dc); cudaMemcpy(&hc, dc, 8, cudaMemcpyDeviceToHost);
        printf("BAR + STS/LDS round, %3d thr %.1f cycles\n", nt, (double)hc / N);
    }
    k_rcp<<<1, 32>>>(dd, dc, 3.0); cudaMemcpy(&hc, dc, 8, cudaMemcpyDeviceToHost);
    printf("1.0/x (+DADD) latency         %.1f cycles\n", (double)hc / N);
    for (int w : {1, 4, 8, 16}) {
        k_dfma_tput<<<1, 32 * w>>>(dd, dc, 1.0000001, 1e-9); cudaMemcpy(&hc, dc, 8, cudaMemcpyDeviceToHost);
        printf("DFMA throughput, %2d warps    %.2f cycles per warp-DFMA per SM\n", w, (double)hc / (N * 8.0 * w));
    }
    return 0;
}

// ---- FP64 tensor core (mma.sync m8n8k4 f64 -> SASS DMMA) throughput
__global__ void k_dmma(double *out, long long *cyc) {
    double a = threadIdx.x * 1e-3, b = 1.0 + threadIdx.x * 1e-4;
    double c[8][2];
    for (int j = 0; j < 8; ++j) { c[j][0] = 0; c[j][1] = 0; }
    long long t0 = clock64();
    for (int i = 0; i < N; ++i) {
#pragma unroll
        for (int j = 0; j < 8; ++j)
            asm volatile("mma.sync.aligned.m8n8k4.row.col.f64.f64.f64.f64 {%0,%1}, {%2}, {%3}, {%0,%1};\n"
                         : "+d"(c[j][0]), "+d"(c[j][1]) : "d"(a), "d"(b));
    }
    long long t1 = clock64();
    double s = 0;
    for (int j = 0; j < 8; ++j) s += c[j][0] + c[j][1];
    out[blockIdx.x * blockDim.x + threadIdx.x] = s;
    if (threadIdx.x == 0 && blockIdx.x == 0) cyc[0] = t1 - t0;
}

int main2() {
    double *dd; long long *dc; long long hc;
    cudaMalloc(&dd, 1 << 22); cudaMalloc(&dc, 64);
    for (int w : {1, 4, 8, 16}) {
        k_dmma<<<1, 32 * w>>>(dd, dc); cudaMemcpy(&hc, dc, 8, cudaMemcpyDeviceToHost);
        double per = (double)hc / (N * 8.0 * w);
        printf("DMMA m8n8k4, %2d warps: %.2f cycles per warp-mma per SM -> %.0f FMA/clk/SM\n", w, per, 256.0 / per);
    }
    return 0;
}
int main() { main1(); return main2(); }

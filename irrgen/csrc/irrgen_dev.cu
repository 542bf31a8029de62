// irrgen_dev.cu -- device-side copy of the seeded value generator of
// irrgen/__init__.py (SURVEY §8(d) "Generators"): input construction only,
// none of the method's arithmetic.  Used where the host cannot build the
// batch (C5: 200,000 fronts, 68 GB), so each rank generates its own matrices
// in HBM, keyed by GLOBAL id exactly as the host generator:
//     key  = splitmix64(seed ^ splitmix64(gid))
//     a_ij = 2 * ((splitmix64(key + (i + j*m)) >> 11) * 2^-53) - 1
// (an exact dyadic in [-1, 1); a test asserts byte equality with the host).
#include <cuda_runtime.h>
#include <stdint.h>

namespace {

__device__ __forceinline__ uint64_t splitmix64(uint64_t x) {
    uint64_t z = x + 0x9E3779B97F4A7C15ull;
    z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ull;
    z = (z ^ (z >> 27)) * 0x94D049BB133111EBull;
    return z ^ (z >> 31);
}

// one CTA per matrix (grid-stride over matrices), threads over i + j*m
__global__ void __launch_bounds__(256) fill_kernel(int count, const int *__restrict__ m, const int *__restrict__ n,
                                                   const int *__restrict__ ld, const long long *__restrict__ off,
                                                   const long long *__restrict__ gid, unsigned long long seed,
                                                   double *__restrict__ out) {
    for (int g = blockIdx.x; g < count; g += gridDim.x) {
        const int mg = m[g], ng = n[g], lg = ld[g];
        const uint64_t key = splitmix64(seed ^ splitmix64((uint64_t)gid[g]));
        double *o = out + off[g];
        if (lg == mg) {
            const long long tot = (long long)mg * ng;
            for (long long e = threadIdx.x; e < tot; e += blockDim.x) {
                const uint64_t x = splitmix64(key + (uint64_t)e);
                o[e] = 2.0 * ((double)(x >> 11) * 0x1p-53) - 1.0;
            }
        } else {
            for (int j = 0; j < ng; ++j)
                for (int i = threadIdx.x; i < mg; i += blockDim.x) {
                    const uint64_t x = splitmix64(key + (uint64_t)i + (uint64_t)j * (uint64_t)mg);
                    o[i + (long long)j * lg] = 2.0 * ((double)(x >> 11) * 0x1p-53) - 1.0;
                }
        }
    }
}

}  // namespace

extern "C" {

// Fill matrix g (m[g] x n[g], leading dimension ld[g]) at out + off[g] with
// the value stream of global id gid[g].  All arrays are device memory; count
// matrices; asynchronous on `stream`.  Returns 0, or the CUDA error code.
int irrgen_fill_device(int count, const int *m, const int *n, const int *ld, const long long *off,
                       const long long *gid, unsigned long long seed, double *out, cudaStream_t stream) {
    if (count <= 0) return 0;
    int dev = 0, sms = 148;
    cudaGetDevice(&dev);
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
    int grid = sms * 8;
    if (grid > count) grid = count;
    fill_kernel<<<grid, 256, 0, stream>>>(count, m, n, ld, off, gid, seed, out);
    return (int)cudaGetLastError();
}

}

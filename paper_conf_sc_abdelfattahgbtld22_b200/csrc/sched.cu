// sched.cu -- device counting sort of a batch by a size key (see sched.cuh).
#include "sched.cuh"

namespace irr {

__global__ void size_hist_kernel(const int *key, int batch, int *counts) {
    __shared__ int h[SORT_BUCKETS];
    for (int b = threadIdx.x; b < SORT_BUCKETS; b += blockDim.x) h[b] = 0;
    __syncthreads();
    for (int i = blockIdx.x * blockDim.x + threadIdx.x; i < batch; i += gridDim.x * blockDim.x)
        atomicAdd(&h[size_bucket(key[i])], 1);
    __syncthreads();
    for (int b = threadIdx.x; b < SORT_BUCKETS; b += blockDim.x)
        if (h[b]) atomicAdd(&counts[b], h[b]);
}

// prefix[b] = #entries with bucket >= b; cursor[b] = start of bucket b in the
// descending order (= prefix[b+1])
__global__ void size_scan_kernel(int *counts, int *prefix, int *cursor) {
    if (threadIdx.x != 0) return;
    int acc = 0;
    prefix[SORT_BUCKETS] = 0;
    for (int b = SORT_BUCKETS - 1; b >= 0; --b) {
        cursor[b] = acc;
        acc += counts[b];
        prefix[b] = acc;
    }
}

__global__ void size_scatter_kernel(const int *key, int batch, int *cursor, int *sorted) {
    const int i = blockIdx.x * blockDim.x + threadIdx.x;
    if (i >= batch) return;
    sorted[atomicAdd(&cursor[size_bucket(key[i])], 1)] = i;
}

void launch_size_sort(const int *key, int batch, int *ws, cudaStream_t s) {
    int *sorted = ws;
    int *prefix = ws + batch;
    int *counts = prefix + SORT_BUCKETS + 1;
    int *cursor = counts + SORT_BUCKETS + 1;
    cudaMemsetAsync(counts, 0, (SORT_BUCKETS + 1) * sizeof(int), s);
    int grid = (batch + 255) / 256;
    if (grid > 1024) grid = 1024;
    if (grid < 1) grid = 1;
    {
        KScope k(K_MISC, s);
        size_hist_kernel<<<grid, 256, 0, s>>>(key, batch, counts);
    }
    {
        KScope k(K_MISC, s);
        size_scan_kernel<<<1, 32, 0, s>>>(counts, prefix, cursor);
    }
    {
        KScope k(K_MISC, s);
        size_scatter_kernel<<<(batch + 255) / 256, 256, 0, s>>>(key, batch, cursor, sorted);
    }
}

}  // namespace irr

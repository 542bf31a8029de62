// sched.cuh -- device-side work scheduling shared by the building blocks.
//
// DCWI decides per matrix how much work a call has; on a batch
// of 50,000 fronts where only a handful are large, a grid sized for the
// required dims spends its time skipping empty matrices.  Instead:
//   * scan_units_kernel: one CTA turns per-slot work-unit counts into prefix
//     offsets (tile_off[0..count]);
//   * walk: every persistent CTA takes a contiguous range of the global unit
//     index space, finds its first slot by one binary search and walks on;
//   * SizeSort: a device counting sort of the matrices by a size key
//     (descending buckets of 32) so a call that only concerns matrices with
//     key > t scans just the prefix of the sorted list (TRSM recursion levels).
#pragma once
#include "irr_internal.cuh"

namespace irr {

constexpr int SORT_BUCKETS = 130;  // key / 32 capped at 129

struct SlotList {
    const int *idx;        // slot -> matrix (nullptr: identity)
    const int *prefix;     // prefix[b] = #entries with bucket >= b (nullptr: use count)
    int bucket0;           // active prefix = prefix[bucket0]
    __device__ __forceinline__ int matrix(int slot) const { return idx ? idx[slot] : slot; }
    __device__ __forceinline__ int count(int n) const { return prefix ? prefix[bucket0] : n; }
};

inline SlotList all_slots() { return SlotList{nullptr, nullptr, 0}; }

// U: int units(int matrix) const
template <class U>
__global__ void __launch_bounds__(1024) scan_units_kernel(U u, SlotList sl, int n, int *off) {
    __shared__ int warp_sums[32];
    __shared__ int carry_s;
    const int count = sl.count(n);
    const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
    if (tid == 0) carry_s = 0;
    __syncthreads();
    for (int base = 0; base < count; base += 1024) {
        const int b = base + tid;
        const int v = (b < count) ? u.units(sl.matrix(b)) : 0;
        int x = v;
#pragma unroll
        for (int o = 1; o < 32; o <<= 1) {
            int y = __shfl_up_sync(FULL, x, o);
            if (lane >= o) x += y;
        }
        if (lane == 31) warp_sums[warp] = x;
        __syncthreads();
        if (warp == 0) {
            int w = warp_sums[lane];
#pragma unroll
            for (int o = 1; o < 32; o <<= 1) {
                int y = __shfl_up_sync(FULL, w, o);
                if (lane >= o) w += y;
            }
            warp_sums[lane] = w;
        }
        __syncthreads();
        const int excl = carry_s + (warp ? warp_sums[warp - 1] : 0) + x - v;
        if (b < count) off[b] = excl;
        __syncthreads();
        if (tid == 1023) carry_s = excl + v;
        __syncthreads();
    }
    if (tid == 0) off[count] = carry_s;
}

// Contiguous range walk: calls f(matrix, local_unit) for this CTA's units.
// All threads of the CTA call it; f is executed by the whole CTA.
template <class F>
__device__ __forceinline__ void walk_units(const SlotList &sl, int n, const int *__restrict__ off, F f) {
    const int count = sl.count(n);
    if (count <= 0) return;
    const int total = off[count];
    const long long G = gridDim.x;
    const int t0 = (int)((long long)blockIdx.x * total / G);
    const int t1 = (int)((long long)(blockIdx.x + 1) * total / G);
    if (t0 >= t1) return;
    int lo = 0, hi = count - 1;
    while (lo < hi) {
        int mid = (lo + hi + 1) >> 1;
        if (off[mid] <= t0) lo = mid; else hi = mid - 1;
    }
    int b = lo, b_beg = off[b], b_end = off[b + 1];
    for (int t = t0; t < t1; ++t) {
        while (t >= b_end) {
            ++b;
            b_beg = off[b];
            b_end = off[b + 1];
        }
        f(sl.matrix(b), t - b_beg);
    }
}

// ---------------------------------------------------------------- size sort
// keys: int[batch]; order: descending buckets of 32.  counts/prefix: int[SORT_BUCKETS+1]
__global__ void size_hist_kernel(const int *key, int batch, int *counts);
__global__ void size_scan_kernel(int *counts, int *prefix, int *cursor);
__global__ void size_scatter_kernel(const int *key, int batch, int *cursor, int *sorted);

__host__ __device__ inline int size_bucket(int k) {
    int b = k > 0 ? (k >> 5) : 0;
    return b < SORT_BUCKETS - 1 ? b : SORT_BUCKETS - 1;
}

// work space needed by launch_size_sort (ints)
inline size_t size_sort_ints(int batch) { return (size_t)batch + 3 * (SORT_BUCKETS + 1); }
// sorted = ws[0..batch), prefix = ws + batch (+SORT_BUCKETS+1 entries)
void launch_size_sort(const int *key, int batch, int *ws, cudaStream_t s);
inline SlotList sorted_slots(int *ws, int batch, int min_key_exclusive) {
    return SlotList{ws, ws + batch, size_bucket(min_key_exclusive + 1)};
}

}  // namespace irr

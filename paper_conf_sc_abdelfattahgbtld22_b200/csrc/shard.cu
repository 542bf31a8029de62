// shard.cu -- host-side flop-balanced partition of a batch over the GPUs of
// one box (north_star: "fronts are partitioned flop-balanced
// across the GPUs").  Host code only: the matrices are independent, so the
// partition is the whole multi-GPU plan; the only collective is the gather of
// the status words (irr_status_words).
#include <algorithm>
#include <cmath>
#include <numeric>
#include <queue>
#include <vector>

#include "irr.h"

namespace {
// LAPACK / MAGMA FLOPS_DGETRF (SURVEY reading Q1)
double getrf_flops(double m, double n) {
    const double big = m > n ? m : n, k = m < n ? m : n;
    if (k <= 0) return 0.0;
    return big * k * k - k * k * k / 3.0 - k * k / 2.0 + 5.0 * k / 6.0;
}
}  // namespace

extern "C" {

int irr_shard_lpt_work(int batch, const double *work, int parts, int *owner) {
    if (batch < 0) return -1;
    if (batch > 0 && !work) return -2;
    if (parts < 1) return -3;
    if (batch > 0 && !owner) return -4;
    // longest processing time first: by work descending, index ascending; each
    // item to the least-loaded part (ties -> lowest part id)
    std::vector<int> order(batch);
    std::iota(order.begin(), order.end(), 0);
    std::stable_sort(order.begin(), order.end(), [&](int a, int b) { return work[a] > work[b]; });
    using Slot = std::pair<double, int>;
    std::priority_queue<Slot, std::vector<Slot>, std::greater<Slot>> heap;
    for (int p = 0; p < parts; ++p) heap.push({0.0, p});
    for (int i : order) {
        Slot s = heap.top();
        heap.pop();
        owner[i] = s.second;
        heap.push({s.first + work[i], s.second});
    }
    return IRR_SUCCESS;
}

int irr_shard_lpt(int batch, const int *m, const int *n, int parts, int *owner) {
    if (batch < 0) return -1;
    if (batch > 0 && (!m || !n)) return -2;
    if (parts < 1) return -4;
    if (batch > 0 && !owner) return -5;
    std::vector<double> w(batch);
    for (int i = 0; i < batch; ++i) w[i] = getrf_flops(m[i], n[i]);
    return irr_shard_lpt_work(batch, w.data(), parts, owner);
}

}  // extern "C"

// api.cu -- the C ABI entry points (include/irr.h) and the host drivers.
//
// The host side only checks scalar arguments, carves the caller's workspace
// and enqueues kernels; it never touches per-matrix data (the
// expanded interface exists so that no pointer/size arithmetic runs on the
// host).  The only host loop is over panel ITERATIONS of the largest matrix
// (P:L167, L179).
#include <algorithm>
#include <cstring>
#include <cstdlib>
#include <map>
#include <mutex>
#include <vector>

#include "irr_internal.cuh"
#include "sched.cuh"

namespace irr {

void launch_gemm_masked(const GemmArgs &g, const int *mask, int *counters, int *tile_off, cudaStream_t s,
                        SlotList sl);
void run_trsm_masked(const TrsmArgs &t, const int *mask, int *counters, int *tile_off, cudaStream_t s,
                     int *sort_ws);
void launch_laswp_masked(int max_n, const int *n, double *const *A, int Ai, int Aj, const int *lda, int k1, int k2,
                         const int *kcount, int *const *ipiv, int batch, const int *mask, cudaStream_t s,
                         int *units_off, SlotList sl);
size_t laswp_smem(int span);
bool getrs_strip_ok(int max_n1);
bool getrs_vec_ok(int max_n, int max_nrhs);
void launch_getrs_vec(int batch, int max_n, int max_nrhs, const int *n, const int *nrhs, const double *const *A,
                      const int *lda, int *const *ipiv, double *const *B, const int *ldb, const int *mask,
                      cudaStream_t s);
void launch_getrs_strip(int batch, const int *n1, const int *n2, const double *const *F11, const int *ld11,
                        double *const *F12, const int *ld12, int *const *ipiv, const int *info, int *units_off,
                        int *queue, SlotList sl, cudaStream_t s, int upper = 1);

// defaults chosen by measurement on B200: tier M only up to
// 48 KB (C2 6.20 -> 6.06 ms against 96 KB, once L1 got faster; C4 100.5 ->
// 100.4; 0 = no tier M is 6.00 on C2 but slower on C5), S/M concurrent with L1, DMMA for the
// grid-wide GEMMs (22.1 vs 17.5 TFLOP/s) and inside L1 (C2 6.53 -> 6.44 ms once
// the deferred interchanges took the L1 kernel off its spills), deferred L1
// left-block interchanges (6.80 -> 6.53 ms), two-level grid tier with outer
// blocks of 128 (round 2: C5 747 -> 637 ms, C3 59.9 -> 57.7 ms; 64 / 96 slower),
// CTA-per-matrix tier up to 512 rows (C5 641 -> 629, C3 57.5 -> 56.2 ms; 1024
// rows: C3 61.7), warp-specialised xgemm (8 DMMA warps + a producer warpgroup on an
// mbarrier ring: C5 616 -> 572 ms, C3 54.8 -> 52.0, C4 91.8 -> 87.0; 16 warps: C3 58.3, C5 651 ms),
// its A operand by TMA bulk copies (C5 576.7 -> 575.8, C3 52.22 -> 52.18 ms: neutral, kept;
// ring 5 x 16: C5 598, 3 x 32: 630 ms); few-large batches (<= 32 matrices) with the
// inner trailing update as a grid-wide GEMM (one 4096^2 matrix 50.7 -> 41.1 ms, 8 of them 72.4 -> 58.2).
static Tuning g_default = {32, 2, M1_ELEMS, 768, 32, 1, 0, 3, 1, 1, 1, 1, 1, 1, 0, 1, 512, 1, 1, NB_OUTER_MAX, 9, 1, 1, 64, 1, 0, 2};
static Tuning g_tuning = g_default;
Tuning &tuning() { return g_tuning; }

long long &launch_counter() {
    static thread_local long long c = 0;
    return c;
}

// ---------------------------------------------------------------- profiling
// Optional per-kernel-class device timing for the benchmark: each launch is
// bracketed by two CUDA events on its own stream (pool created on enable,
// never on the hot path).
static bool g_prof = false;
struct ProfRec { int cls; int ev0, ev1; };
static std::vector<cudaEvent_t> g_events;
static std::vector<ProfRec> g_recs;
static size_t g_ev_used = 0;
static std::vector<int> g_open;  // stack of open record indices

bool prof_on() { return g_prof; }

void prof_record(int cls, cudaStream_t s, bool begin) {
    if (g_ev_used >= g_events.size()) return;  // pool exhausted: stop recording
    if (begin) {
        int e = (int)g_ev_used++;
        cudaEventRecord(g_events[e], s);
        g_recs.push_back({cls, e, -1});
        g_open.push_back((int)g_recs.size() - 1);
    } else {
        if (g_open.empty()) return;
        int r = g_open.back();
        g_open.pop_back();
        int e = (int)g_ev_used++;
        cudaEventRecord(g_events[e], s);
        g_recs[r].ev1 = e;
    }
}

static const char *k_names[NKCLASS] = {"classify", "lu_small", "lu_mid", "panel", "swap_trsm", "gemm_scan",
                                       "gemm_trailing", "trsm_leaf", "gemm_dcwi", "laswp", "misc", "lu_l1", "strip", "getrs", "extend_add",
                                       "zgetrf", "outer_trsm", "left_swaps"};

struct DeviceInfo {
    int sms = 0;
    int major = 0, minor = 0;
    size_t smem_optin = 0;
};
static DeviceInfo g_dev[64];
static std::mutex g_dev_mu;

static const DeviceInfo *device_info() {
    int dev = 0;
    if (cudaGetDevice(&dev) != cudaSuccess || dev < 0 || dev >= 64) return nullptr;
    std::lock_guard<std::mutex> lk(g_dev_mu);
    DeviceInfo &d = g_dev[dev];
    if (d.sms == 0) {
        cudaDeviceProp p;
        if (cudaGetDeviceProperties(&p, dev) != cudaSuccess) return nullptr;
        d.sms = p.multiProcessorCount;
        d.major = p.major;
        d.minor = p.minor;
        d.smem_optin = p.sharedMemPerBlockOptin;
    }
    return &d;
}

cudaError_t smem_optin_fn(const void *func, size_t bytes) {
    int dev = 0;
    cudaError_t e = cudaGetDevice(&dev);
    if (e != cudaSuccess) return e;
    static std::mutex mu;
    static std::map<std::pair<const void *, int>, size_t> done;
    std::lock_guard<std::mutex> lk(mu);
    size_t &have = done[{func, dev}];
    if (have >= bytes) return cudaSuccess;
    e = cudaFuncSetAttribute(func, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)bytes);
    if (e == cudaSuccess) have = bytes;
    return e;
}

int num_sms() {
    const DeviceInfo *d = device_info();
    return d ? d->sms : 148;
}

// Per-device side stream + fork/join events, created once (never on the hot
// path after the first call).  Non-blocking w.r.t. the legacy stream.
struct DeviceStreams {
    cudaStream_t side = nullptr;
    cudaEvent_t fork = nullptr, join = nullptr;
    cudaStream_t side2 = nullptr;             // the grid tier's second part
    cudaEvent_t fork2 = nullptr, join2 = nullptr;
    cudaStream_t side3 = nullptr;             // tier S: the narrow classes beside the wide ones
    cudaEvent_t fork3 = nullptr, join3 = nullptr;
};
static DeviceStreams g_streams[64];

static DeviceStreams *dev_streams() {
    int dev = 0;
    if (cudaGetDevice(&dev) != cudaSuccess || dev < 0 || dev >= 64) return nullptr;
    std::lock_guard<std::mutex> lk(g_dev_mu);
    DeviceStreams &d = g_streams[dev];
    if (!d.side) {
        if (cudaStreamCreateWithFlags(&d.side, cudaStreamNonBlocking) != cudaSuccess) { d.side = nullptr; return nullptr; }
        cudaEventCreateWithFlags(&d.fork, cudaEventDisableTiming);
        cudaEventCreateWithFlags(&d.join, cudaEventDisableTiming);
        if (cudaStreamCreateWithFlags(&d.side2, cudaStreamNonBlocking) != cudaSuccess) d.side2 = nullptr;
        cudaEventCreateWithFlags(&d.fork2, cudaEventDisableTiming);
        cudaEventCreateWithFlags(&d.join2, cudaEventDisableTiming);
        if (cudaStreamCreateWithFlags(&d.side3, cudaStreamNonBlocking) != cudaSuccess) d.side3 = nullptr;
        cudaEventCreateWithFlags(&d.fork3, cudaEventDisableTiming);
        cudaEventCreateWithFlags(&d.join3, cudaEventDisableTiming);
    }
    return &d;
}
static cudaStream_t side_stream() {
    DeviceStreams *d = dev_streams();
    return d ? d->side : nullptr;
}
static cudaEvent_t fork_event() { return dev_streams()->fork; }
static cudaEvent_t join_event() { return dev_streams()->join; }

static int check_device() {
    const DeviceInfo *d = device_info();
    if (!d) return IRR_ERR_CUDA;
    if (d->major != 10 || d->minor != 0) return IRR_ERR_DEVICE;  // built for sm_100a only
    return IRR_SUCCESS;
}

// ---------------------------------------------------------------- workspace
struct Work {
    int *counters;
    int *bins;
    int *tile_off;
    int *sort;  // size sort (sched.cuh): sorted slots + bucket prefix
    int *keys;  // per-matrix sort keys
    void *plans;  // getrf / partial only: one interchange plan per tier-L slot
    void *outer_plans;  // getrf / partial only: one outer-block plan per tier-L slot (two-level tier)
    int *part_counters, *part_list, *part_tile_off;  // getrf / partial only: the grid tier's second part
};

static size_t work_bytes_for(int batch) {
    size_t b = (size_t)(batch > 0 ? batch : 1);
    return align256(CNT_INTS * sizeof(int)) + align256(NBINS * b * sizeof(int)) + align256((b + 1) * sizeof(int)) +
           align256(size_sort_ints((int)b) * sizeof(int)) + align256(b * sizeof(int));
}

// getrf / partial: the common part plus the per-slot interchange plans of the
// grid-wide tier (written by its panel kernel, read by its strip kernel)
static size_t work_bytes_getrf(int batch) {
    size_t b = (size_t)(batch > 0 ? batch : 1);
    return work_bytes_for(batch) + align256(b * SWAP_PLAN_BYTES) + align256(b * OUTER_PLAN_BYTES) +
           align256(CNT_INTS * sizeof(int)) + align256(b * sizeof(int)) + align256((b + 1) * sizeof(int));
}

static Work carve(void *work, int batch) {
    size_t b = (size_t)(batch > 0 ? batch : 1);
    char *p = (char *)work;
    Work w;
    w.counters = (int *)p;
    p += align256(CNT_INTS * sizeof(int));
    w.bins = (int *)p;
    p += align256(NBINS * b * sizeof(int));
    w.tile_off = (int *)p;
    p += align256((b + 1) * sizeof(int));
    w.sort = (int *)p;
    p += align256(size_sort_ints((int)b) * sizeof(int));
    w.keys = (int *)p;
    p += align256(b * sizeof(int));
    w.plans = p;  // valid only in a work_bytes_getrf() workspace
    p += align256(b * SWAP_PLAN_BYTES);
    w.outer_plans = p;
    p += align256(b * OUTER_PLAN_BYTES);
    w.part_counters = (int *)p;
    p += align256(CNT_INTS * sizeof(int));
    w.part_list = (int *)p;
    p += align256(b * sizeof(int));
    w.part_tile_off = (int *)p;
    return w;
}

static int resolve_max_dims(int batch, int &max_m, int &max_n, const int *m, const int *n, int *counters,
                            cudaStream_t s) {
    if (max_m > 0 && max_n > 0) return IRR_SUCCESS;
    IRR_CUDA_TRY(cudaMemsetAsync(counters, 0, CNT_INTS * sizeof(int), s));
    launch_max_dims(batch, m, n, counters, s);
    int h[2];
    IRR_CUDA_TRY(cudaMemcpyAsync(h, counters + CNT_MAXM, 2 * sizeof(int), cudaMemcpyDeviceToHost, s));
    IRR_CUDA_TRY(cudaStreamSynchronize(s));
    if (max_m <= 0) max_m = h[0];
    if (max_n <= 0) max_n = h[1];
    return IRR_SUCCESS;
}

// Enqueue the whole getrf machinery for the (already validated) args.
static int getrf_core(const GetrfArgs &a, const Work &w, int keep_neg_info, cudaStream_t s) {
    IRR_CUDA_TRY(cudaMemsetAsync(w.counters, 0, CNT_INTS * sizeof(int), s));
    launch_classify(a, w.counters, w.bins, keep_neg_info, s);
    if (a.max_m <= 0 || a.max_n <= 0) return cudaGetLastError() == cudaSuccess ? IRR_SUCCESS : IRR_ERR_CUDA;
    const Tuning &t = tuning();
    // which tiers can be populated, from the required dims alone
    const long long big = (long long)mid_lds(a.max_m) * a.max_n;
    const bool only_s = t.tier_s && a.max_m <= 32 && a.max_n <= 32;
    const long long mmax = t.tier_m_max;
    const bool has_large = !only_s && big > mmax;
    // The tiers touch disjoint matrices: with a large tier present, S and M run
    // on a forked stream concurrently with it (fills each other's tails).
    cudaStream_t side = s;
    if (has_large && t.concurrent) {
        side = side_stream();
        if (side) {
            IRR_CUDA_TRY(cudaEventRecord(fork_event(), s));
            IRR_CUDA_TRY(cudaStreamWaitEvent(side, fork_event(), 0));
        } else {
            side = s;
        }
    }
    if (t.tier_s) {
        // batches of tier-S matrices only: the narrow classes on a second
        // stream fill the wide classes' tails (C1big 3.44 -> 3.30 ms); with
        // larger tiers present, tier S already runs beside them on `side`
        DeviceStreams *ds = (t.concurrent && only_s) ? dev_streams() : nullptr;
        SmallStreams ss{ds ? ds->side3 : nullptr, ds ? ds->fork3 : nullptr, ds ? ds->join3 : nullptr};
        launch_lu_small(a, w.counters, w.bins, side, ss.s2 ? &ss : nullptr);
    }
    if (!only_s) {
        if (mmax > 0) {
            launch_lu_mid(a, w.counters, w.bins, BIN_M1, (int)(mmax < M1_ELEMS ? mmax : M1_ELEMS), side);
            if (big > M1_ELEMS && mmax > M1_ELEMS)
                launch_lu_mid(a, w.counters, w.bins, BIN_M2, (int)(mmax < M2_ELEMS ? mmax : M2_ELEMS), side);
            if (big > M2_ELEMS && mmax > M2_ELEMS) launch_lu_mid(a, w.counters, w.bins, BIN_M3, (int)mmax, side);
        }
        if (has_large) {
            if (t.l1) launch_lu_l1(a, w.counters, w.bins, w.keys, w.sort, s);
            if (!t.l1 || a.max_m > t.l1_rows) {
                DeviceStreams *ds = dev_streams();
                PartWork pw{w.part_counters, w.part_list, w.part_tile_off, ds ? ds->side2 : nullptr,
                            ds ? ds->fork2 : nullptr, ds ? ds->join2 : nullptr};
                launch_lu_large(a, w.counters, w.bins, w.tile_off, w.plans, w.outer_plans, s, w.keys, w.sort, &pw);
            }
        }
    }
    if (side != s) {
        IRR_CUDA_TRY(cudaEventRecord(join_event(), side));
        IRR_CUDA_TRY(cudaStreamWaitEvent(s, join_event(), 0));
    }
    return cudaGetLastError() == cudaSuccess ? IRR_SUCCESS : IRR_ERR_CUDA;
}

}  // namespace irr

using namespace irr;

extern "C" {

const char *irr_version(void) { return "irrlu-b200 0.1 (sm_100a)"; }

int irr_profile_enable(int max_launches) {
    for (cudaEvent_t e : g_events) cudaEventDestroy(e);
    g_events.clear();
    g_recs.clear();
    g_open.clear();
    g_ev_used = 0;
    g_prof = max_launches > 0;
    if (!g_prof) return IRR_SUCCESS;
    g_events.resize((size_t)max_launches * 2);
    for (auto &e : g_events)
        if (cudaEventCreate(&e) != cudaSuccess) { g_prof = false; return IRR_ERR_CUDA; }
    return IRR_SUCCESS;
}

int irr_profile_collect(double *ms, long long *launches, int nclass) {
    for (int c = 0; c < nclass; ++c) { ms[c] = 0.0; launches[c] = 0; }
    int n = 0;
    for (const ProfRec &r : g_recs) {
        if (r.ev1 < 0 || r.cls >= nclass) continue;
        if (cudaEventSynchronize(g_events[r.ev1]) != cudaSuccess) return -1;
        float t = 0.f;
        cudaEventElapsedTime(&t, g_events[r.ev0], g_events[r.ev1]);
        ms[r.cls] += t;
        launches[r.cls] += 1;
        ++n;
    }
    g_recs.clear();
    g_open.clear();
    g_ev_used = 0;
    return n;
}

int irr_profile_busy(double *busy_ms, int nclass) {
    for (int c = 0; c < nclass; ++c) busy_ms[c] = 0.0;
    int base = -1;
    std::vector<std::pair<int, std::pair<double, double>>> iv;  // (class, [t0, t1]) in ms from the first launch
    for (const ProfRec &r : g_recs) {
        if (r.ev1 < 0 || r.cls >= nclass) continue;
        if (cudaEventSynchronize(g_events[r.ev1]) != cudaSuccess) return -1;
        if (base < 0) base = r.ev0;
        float t0 = 0.f, t1 = 0.f;
        if (cudaEventElapsedTime(&t0, g_events[base], g_events[r.ev0]) != cudaSuccess) return -1;
        if (cudaEventElapsedTime(&t1, g_events[base], g_events[r.ev1]) != cudaSuccess) return -1;
        iv.push_back({r.cls, {(double)t0, (double)t1}});
    }
    std::sort(iv.begin(), iv.end());
    for (size_t a = 0; a < iv.size();) {  // merge the overlapping intervals of each class
        const int c = iv[a].first;
        double lo = iv[a].second.first, hi = iv[a].second.second;
        size_t b = a + 1;
        for (; b < iv.size() && iv[b].first == c; ++b) {
            if (iv[b].second.first > hi) {
                busy_ms[c] += hi - lo;
                lo = iv[b].second.first;
                hi = iv[b].second.second;
            } else if (iv[b].second.second > hi) {
                hi = iv[b].second.second;
            }
        }
        busy_ms[c] += hi - lo;
        a = b;
    }
    return (int)iv.size();
}

int irr_profile_num_classes(void) { return NKCLASS; }

const char *irr_profile_class_name(int c) { return (c >= 0 && c < NKCLASS) ? k_names[c] : ""; }

long long irr_launch_count(int reset) {
    long long c = launch_counter();
    if (reset) launch_counter() = 0;
    return c;
}

void irr_set_tuning(const char *key, int value) {
    if (!key) return;
    if (!strcmp(key, "nb")) g_tuning.nb = value < 1 ? 1 : (value > 64 ? 64 : value);
    else if (!strcmp(key, "tier_s")) g_tuning.tier_s = value < 0 ? 0 : (value > 2 ? 2 : value);
    else if (!strcmp(key, "tier_m_max")) g_tuning.tier_m_max = value < 0 ? 0 : (value > TIER_M_MAX_DEFAULT ? TIER_M_MAX_DEFAULT : value);
    else if (!strcmp(key, "panel_rows")) g_tuning.panel_rows = value < 0 ? 0 : value;
    else if (!strcmp(key, "trsm_nb")) g_tuning.trsm_nb = value < 1 ? 1 : (value > 32 ? 32 : value);
    else if (!strcmp(key, "l1")) g_tuning.l1 = value ? 1 : 0;
    else if (!strcmp(key, "phase_timing")) g_tuning.phase_timing = value ? 1 : 0;
    else if (!strcmp(key, "l1_ctas_per_sm")) g_tuning.l1_ctas_per_sm = value < 1 ? 1 : (value > 3 ? 3 : value);
    else if (!strcmp(key, "concurrent")) g_tuning.concurrent = value ? 1 : 0;
    else if (!strcmp(key, "dmma")) g_tuning.dmma = value ? 1 : 0;
    else if (!strcmp(key, "l1_dmma")) g_tuning.l1_dmma = value ? 1 : 0;
    else if (!strcmp(key, "panel_win")) g_tuning.panel_win = value ? 1 : 0;
    else if (!strcmp(key, "strip")) g_tuning.strip = value ? 1 : 0;
    else if (!strcmp(key, "gemm_big")) g_tuning.gemm_big = value ? 1 : 0;
    else if (!strcmp(key, "getrs_fused")) g_tuning.getrs_fused = value ? 1 : 0;
    else if (!strcmp(key, "getrs_vec")) g_tuning.getrs_vec = value ? 1 : 0;
    else if (!strcmp(key, "l1_rows")) g_tuning.l1_rows = value < 1 ? 1 : (value > L1_TALL_ROWS ? L1_TALL_ROWS : value);
    else if (!strcmp(key, "defer") || !strcmp(key, "l1_defer")) g_tuning.defer = value ? 1 : 0;
    else if (!strcmp(key, "nb_outer")) g_tuning.nb_outer = value < 0 ? 0 : (value > NB_OUTER_MAX ? NB_OUTER_MAX : value);
    else if (!strcmp(key, "xgemm_warps")) g_tuning.xgemm_warps = value >= 16 ? 16 : (value == 9 ? 9 : 8);
    else if (!strcmp(key, "parts")) g_tuning.parts = value >= 2 ? 2 : 1;
    else if (!strcmp(key, "part_grid")) g_tuning.part_grid = value >= 2 ? 2 : 1;
    else if (!strcmp(key, "outer_cols")) g_tuning.outer_cols = value <= 32 ? 32 : 64;
    else if (!strcmp(key, "xgemm_tma")) g_tuning.xgemm_tma = value ? 1 : 0;
    else if (!strcmp(key, "mid_dmma")) g_tuning.mid_dmma = value ? 1 : 0;
    else if (!strcmp(key, "split_strip")) g_tuning.split_strip = value < 0 ? 0 : (value > 2 ? 2 : value);
}

int irr_get_tuning(const char *key) {
    if (!key) return -1;
    if (!strcmp(key, "nb")) return g_tuning.nb;
    if (!strcmp(key, "tier_s")) return g_tuning.tier_s;
    if (!strcmp(key, "tier_m_max")) return g_tuning.tier_m_max;
    if (!strcmp(key, "panel_rows")) return g_tuning.panel_rows;
    if (!strcmp(key, "trsm_nb")) return g_tuning.trsm_nb;
    if (!strcmp(key, "l1")) return g_tuning.l1;
    if (!strcmp(key, "phase_timing")) return g_tuning.phase_timing;
    if (!strcmp(key, "l1_ctas_per_sm")) return g_tuning.l1_ctas_per_sm;
    if (!strcmp(key, "concurrent")) return g_tuning.concurrent;
    if (!strcmp(key, "dmma")) return g_tuning.dmma;
    if (!strcmp(key, "l1_dmma")) return g_tuning.l1_dmma;
    if (!strcmp(key, "panel_win")) return g_tuning.panel_win;
    if (!strcmp(key, "strip")) return g_tuning.strip;
    if (!strcmp(key, "gemm_big")) return g_tuning.gemm_big;
    if (!strcmp(key, "getrs_fused")) return g_tuning.getrs_fused;
    if (!strcmp(key, "getrs_vec")) return g_tuning.getrs_vec;
    if (!strcmp(key, "l1_rows")) return g_tuning.l1_rows;
    if (!strcmp(key, "defer") || !strcmp(key, "l1_defer")) return g_tuning.defer;
    if (!strcmp(key, "nb_outer")) return g_tuning.nb_outer;
    if (!strcmp(key, "xgemm_warps")) return g_tuning.xgemm_warps;
    if (!strcmp(key, "parts")) return g_tuning.parts;
    if (!strcmp(key, "part_grid")) return g_tuning.part_grid;
    if (!strcmp(key, "outer_cols")) return g_tuning.outer_cols;
    if (!strcmp(key, "xgemm_tma")) return g_tuning.xgemm_tma;
    if (!strcmp(key, "mid_dmma")) return g_tuning.mid_dmma;
    if (!strcmp(key, "split_strip")) return g_tuning.split_strip;
    return -1;
}

void irr_reset_tuning(void) { g_tuning = g_default; }

size_t irr_getrf_workspace_size(int batch, int max_m, int max_n) {
    (void)max_m; (void)max_n;
    return work_bytes_getrf(batch);
}

int irr_getrf(int batch, int max_m, int max_n, const int *m, const int *n, double *const *A, const int *ld,
              int *const *ipiv, int *info, void *work, size_t work_bytes, irr_stream_t stream) {
    if (batch < 0) return -1;
    if (batch == 0) return IRR_SUCCESS;
    if (!m) return -4;
    if (!n) return -5;
    if (!A) return -6;
    if (!ld) return -7;
    if (!ipiv) return -8;
    if (!info) return -9;
    if (!work) return -10;
    if (work_bytes < work_bytes_getrf(batch)) return IRR_ERR_WORKSPACE;
    int rc = check_device();
    if (rc) return rc;
    cudaStream_t s = (cudaStream_t)stream;
    Work w = carve(work, batch);
    rc = resolve_max_dims(batch, max_m, max_n, m, n, w.counters, s);
    if (rc) return rc;
    GetrfArgs a{batch, max_m, max_n, m, n, A, ld, ipiv, info};
    return getrf_core(a, w, 0, s);
}

size_t irr_getrf_partial_workspace_size(int batch, int max_n1, int max_n2) {
    (void)max_n1; (void)max_n2;
    return work_bytes_getrf(batch);
}

}  // extern "C"

namespace irr {
// The partial front factorization, both variants.  lapack == 0: the paper's
// steps: F12 <- U^-1 L^-1 P^T F12, F22 -= F21 F12, F21 untouched.
// lapack == 1: U12 = L^-1 P^T F12, L21 = F21 U^-1,
// F22 -= L21 U12 (F21 overwritten by L21).
static int partial_core(int lapack, int batch, int max_n1, int max_n2, const int *n1, const int *n2,
                        double *const *F11, const int *ld11, double *const *F12, const int *ld12,
                        double *const *F21, const int *ld21, double *const *F22, const int *ld22, int *const *ipiv,
                        int *info, void *work, size_t work_bytes, irr_stream_t stream) {
    if (batch < 0) return -1;
    if (batch == 0) return IRR_SUCCESS;
    if (!n1) return -4;
    if (!n2) return -5;
    if (!F11) return -6;
    if (!ld11) return -7;
    if (!F12) return -8;
    if (!ld12) return -9;
    if (!F21) return -10;
    if (!ld21) return -11;
    if (!F22) return -12;
    if (!ld22) return -13;
    if (!ipiv) return -14;
    if (!info) return -15;
    if (!work) return -16;
    if (work_bytes < work_bytes_getrf(batch)) return IRR_ERR_WORKSPACE;
    int rc = check_device();
    if (rc) return rc;
    cudaStream_t s = (cudaStream_t)stream;
    Work w = carve(work, batch);
    rc = resolve_max_dims(batch, max_n1, max_n2, n1, n2, w.counters, s);
    if (rc) return rc;
    launch_partial_validate(batch, max_n1, max_n2, n1, n2, ld11, ld12, ld21, ld22, F11, F12,
                            (const double *const *)F21, F22, ipiv, info, s);
    // step 1: P L U <- LU(F11), pivoting restricted to F11
    GetrfArgs a{batch, max_n1, max_n1, n1, n1, F11, ld11, ipiv, info};
    rc = getrf_core(a, w, 1, s);
    if (rc) return rc;
    if (max_n1 <= 0 || max_n2 <= 0) return IRR_SUCCESS;
    // fronts sorted by n1 (descending buckets): every building-block call
    // below visits only the fronts that still have work at its offset
    launch_size_sort(n1, batch, w.sort, s);
    TrsmArgs t{};
    t.side = IRR_LEFT; t.uplo = IRR_LOWER; t.trans = IRR_NO_TRANS; t.diag = IRR_UNIT;
    t.max_m = max_n1; t.max_n = max_n2; t.m = n1; t.n = n2; t.alpha = 1.0;
    t.T = (const double *const *)F11; t.Ti = 0; t.Tj = 0; t.ldt = ld11;
    t.B = F12; t.Bi = 0; t.Bj = 0; t.ldb = ld12; t.batch = batch;
    if (tuning().getrs_fused && getrs_strip_ok(max_n1)) {
        // step 2: F12 <- U^-1 L^-1 P^T F12 / U12 <- L^-1 P^T F12: one
        // fused strip kernel (the LAPACK-style variant stops before U^-1)
        launch_getrs_strip(batch, n1, n2, (const double *const *)F11, ld11, F12, ld12, ipiv, info, w.tile_off,
                           w.counters + CNT_GSQ, sorted_slots(w.sort, batch, 0), s, lapack ? 0 : 1);
    } else {
        // irrLASWP + irrTRSM(L, unit) [+ irrTRSM(U)] as the paper composes GETRS
        launch_laswp_masked(max_n2, n2, F12, 0, 0, ld12, 0, max_n1, n1, ipiv, batch, info, s, w.tile_off,
                            sorted_slots(w.sort, batch, 0));
        run_trsm_masked(t, info, w.counters, w.tile_off, s, w.sort);
        if (!lapack) {
            t.uplo = IRR_UPPER; t.diag = IRR_NON_UNIT;
            run_trsm_masked(t, info, w.counters, w.tile_off, s, w.sort);
        }
    }
    if (lapack) {
        // L21 <- F21 U^-1: right side, upper, non-unit (the sort key n1 is the
        // triangular dimension here too)
        TrsmArgs r{};
        r.side = IRR_RIGHT; r.uplo = IRR_UPPER; r.trans = IRR_NO_TRANS; r.diag = IRR_NON_UNIT;
        r.max_m = max_n2; r.max_n = max_n1; r.m = n2; r.n = n1; r.alpha = 1.0;
        r.T = (const double *const *)F11; r.Ti = 0; r.Tj = 0; r.ldt = ld11;
        r.B = F21; r.Bi = 0; r.Bj = 0; r.ldb = ld21; r.batch = batch;
        run_trsm_masked(r, info, w.counters, w.tile_off, s, w.sort);
    }
    // step 3: F22 <- F22 - F21 F12 / F22 - L21 U12
    GemmArgs g{};
    g.ta = 0; g.tb = 0; g.max_m = max_n2; g.max_n = max_n2; g.max_k = max_n1;
    g.m = n2; g.n = n2; g.k = n1; g.alpha = -1.0; g.beta = 1.0;
    g.A = (const double *const *)F21; g.Ai = 0; g.Aj = 0; g.lda = ld21;
    g.B = (const double *const *)F12; g.Bi = 0; g.Bj = 0; g.ldb = ld12;
    g.C = F22; g.Ci = 0; g.Cj = 0; g.ldc = ld22; g.batch = batch;
    launch_gemm_masked(g, info, w.counters, w.tile_off, s, sorted_slots(w.sort, batch, 0));
    return cudaGetLastError() == cudaSuccess ? IRR_SUCCESS : IRR_ERR_CUDA;
}
}  // namespace irr

extern "C" {

int irr_getrf_partial(int batch, int max_n1, int max_n2, const int *n1, const int *n2, double *const *F11,
                      const int *ld11, double *const *F12, const int *ld12, const double *const *F21,
                      const int *ld21, double *const *F22, const int *ld22, int *const *ipiv, int *info, void *work,
                      size_t work_bytes, irr_stream_t stream) {
    return partial_core(0, batch, max_n1, max_n2, n1, n2, F11, ld11, F12, ld12, (double *const *)F21, ld21, F22,
                        ld22, ipiv, info, work, work_bytes, stream);
}

size_t irr_getrf_partial_lapack_workspace_size(int batch, int max_n1, int max_n2) {
    (void)max_n1; (void)max_n2;
    return work_bytes_getrf(batch);
}

int irr_getrf_partial_lapack(int batch, int max_n1, int max_n2, const int *n1, const int *n2, double *const *F11,
                             const int *ld11, double *const *F12, const int *ld12, double *const *F21,
                             const int *ld21, double *const *F22, const int *ld22, int *const *ipiv, int *info,
                             void *work, size_t work_bytes, irr_stream_t stream) {
    return partial_core(1, batch, max_n1, max_n2, n1, n2, F11, ld11, F12, ld12, F21, ld21, F22, ld22, ipiv, info,
                        work, work_bytes, stream);
}

// Step a5.2 of the partial front on its own: X <- U^-1 L^-1 P^T B with the
// factors of irr_getrf (the fused strip kernel, or irrLASWP + 2 x irrTRSM).
static void getrs_core(int batch, int max_n, int max_nrhs, const int *n, const int *nrhs, const double *const *A,
                       const int *lda, int *const *ipiv, double *const *B, const int *ldb, const int *mask,
                       const Work &w, cudaStream_t s) {
    // systems sorted by n (descending buckets): every building-block call
    // visits only the systems that still have work at its offset
    launch_size_sort(n, batch, w.sort, s);
    if (tuning().getrs_fused && getrs_strip_ok(max_n)) {
        launch_getrs_strip(batch, n, nrhs, A, lda, B, ldb, ipiv, mask, w.tile_off, w.counters + CNT_GSQ,
                           sorted_slots(w.sort, batch, 0), s);
        return;
    }
    launch_laswp_masked(max_nrhs, nrhs, B, 0, 0, ldb, 0, max_n, n, ipiv, batch, mask, s, w.tile_off,
                        sorted_slots(w.sort, batch, 0));
    TrsmArgs t{};
    t.side = IRR_LEFT; t.uplo = IRR_LOWER; t.trans = IRR_NO_TRANS; t.diag = IRR_UNIT;
    t.max_m = max_n; t.max_n = max_nrhs; t.m = n; t.n = nrhs; t.alpha = 1.0;
    t.T = A; t.Ti = 0; t.Tj = 0; t.ldt = lda;
    t.B = B; t.Bi = 0; t.Bj = 0; t.ldb = ldb; t.batch = batch;
    run_trsm_masked(t, mask, w.counters, w.tile_off, s, w.sort);
    t.uplo = IRR_UPPER; t.diag = IRR_NON_UNIT;
    run_trsm_masked(t, mask, w.counters, w.tile_off, s, w.sort);
}

size_t irr_getrs_workspace_size(int batch) { return work_bytes_getrf(batch); }

int irr_getrs(irr_trans_t trans, int batch, int max_n, int max_nrhs, const int *n, const int *nrhs,
              const double *const *A, const int *lda, int *const *ipiv, double *const *B, const int *ldb,
              int *info, void *work, size_t work_bytes, irr_stream_t stream) {
    if (trans != IRR_NO_TRANS && trans != IRR_TRANS) return -1;
    if (batch < 0) return -2;
    if (trans == IRR_TRANS) return IRR_ERR_UNSUPPORTED;
    if (batch == 0) return IRR_SUCCESS;
    if (!n) return -5;
    if (!nrhs) return -6;
    if (!A) return -7;
    if (!lda) return -8;
    if (!ipiv) return -9;
    if (!B) return -10;
    if (!ldb) return -11;
    if (!info) return -12;
    if (!work) return -13;
    if (work_bytes < work_bytes_getrf(batch)) return IRR_ERR_WORKSPACE;
    int rc = check_device();
    if (rc) return rc;
    cudaStream_t s = (cudaStream_t)stream;
    Work w = carve(work, batch);
    rc = resolve_max_dims(batch, max_n, max_nrhs, n, nrhs, w.counters, s);
    if (rc) return rc;
    launch_getrs_validate(batch, max_n, max_nrhs, n, nrhs, A, lda, ipiv, B, ldb, info, s);
    if (max_n <= 0 || max_nrhs <= 0) return cudaGetLastError() == cudaSuccess ? IRR_SUCCESS : IRR_ERR_CUDA;
    if (tuning().getrs_vec && getrs_vec_ok(max_n, max_nrhs)) {
        // few right-hand sides (<= GV_MAX_NRHS): CTA per system
        launch_getrs_vec(batch, max_n, max_nrhs, n, nrhs, A, lda, ipiv, B, ldb, info, s);
        return cudaGetLastError() == cudaSuccess ? IRR_SUCCESS : IRR_ERR_CUDA;
    }
    IRR_CUDA_TRY(cudaMemsetAsync(w.counters, 0, CNT_INTS * sizeof(int), s));
    getrs_core(batch, max_n, max_nrhs, n, nrhs, A, lda, ipiv, B, ldb, info, w, s);
    return cudaGetLastError() == cudaSuccess ? IRR_SUCCESS : IRR_ERR_CUDA;
}

int irr_status_words(int batch, const int *m, const int *n, int *const *ipiv, const int *info, unsigned int *words,
                     irr_stream_t stream) {
    if (batch < 0) return -1;
    if (batch == 0) return IRR_SUCCESS;
    if (!m) return -2;
    if (!n) return -3;
    if (!ipiv) return -4;
    if (!info) return -5;
    if (!words) return -6;
    int rc = check_device();
    if (rc) return rc;
    launch_status_words(batch, m, n, ipiv, info, words, (cudaStream_t)stream);
    return cudaGetLastError() == cudaSuccess ? IRR_SUCCESS : IRR_ERR_CUDA;
}

int irr_extend_add(int batch, int max_n2, const int *n2, const double *const *F22, const int *ld22,
                   const int *const *rel, const int *np, double *const *Fp, const int *ldp, int *info,
                   irr_stream_t stream) {
    if (batch < 0) return -1;
    if (max_n2 < 0) return -2;
    if (batch == 0) return IRR_SUCCESS;
    if (!n2) return -3;
    if (!F22) return -4;
    if (!ld22) return -5;
    if (!rel) return -6;
    if (!np) return -7;
    if (!Fp) return -8;
    if (!ldp) return -9;
    if (!info) return -10;
    int rc = check_device();
    if (rc) return rc;
    launch_extend_add(batch, max_n2, n2, F22, ld22, rel, np, Fp, ldp, info, (cudaStream_t)stream);
    return cudaGetLastError() == cudaSuccess ? IRR_SUCCESS : IRR_ERR_CUDA;
}

size_t irr_zgetrf_workspace_size(int batch, int max_m, int max_n) {
    (void)max_m; (void)max_n;
    return work_bytes_for(batch);
}

int irr_zgetrf(int batch, int max_m, int max_n, const int *m, const int *n, double *const *A, const int *ld,
               int *const *ipiv, int *info, void *work, size_t work_bytes, irr_stream_t stream) {
    if (batch < 0) return -1;
    if (batch == 0) return IRR_SUCCESS;
    if (!m) return -4;
    if (!n) return -5;
    if (!A) return -6;
    if (!ld) return -7;
    if (!ipiv) return -8;
    if (!info) return -9;
    if (!work) return -10;
    if (work_bytes < work_bytes_for(batch)) return IRR_ERR_WORKSPACE;
    int rc = check_device();
    if (rc) return rc;
    cudaStream_t s = (cudaStream_t)stream;
    Work w = carve(work, batch);
    rc = resolve_max_dims(batch, max_m, max_n, m, n, w.counters, s);
    if (rc) return rc;
    ZArgs za{batch, max_m, max_n, m, n, A, ld, ipiv, info};
    launch_zgetrf(za, w.counters, w.keys, w.sort, s);
    return cudaGetLastError() == cudaSuccess ? IRR_SUCCESS : IRR_ERR_CUDA;
}

size_t irr_gemm_workspace_size(int batch) { return work_bytes_for(batch); }

int irr_gemm(irr_trans_t ta, irr_trans_t tb, int max_m, int max_n, int max_k, const int *m, const int *n,
             const int *k, double alpha, const double *const *A, int Ai, int Aj, const int *lda,
             const double *const *B, int Bi, int Bj, const int *ldb, double beta, double *const *C, int Ci, int Cj,
             const int *ldc, int batch, void *work, size_t work_bytes, irr_stream_t stream) {
    if (ta != IRR_NO_TRANS && ta != IRR_TRANS) return -1;
    if (tb != IRR_NO_TRANS && tb != IRR_TRANS) return -2;
    if (max_m < 0) return -3;
    if (max_n < 0) return -4;
    if (max_k < 0) return -5;
    if (Ai < 0) return -11;
    if (Aj < 0) return -12;
    if (Bi < 0) return -15;
    if (Bj < 0) return -16;
    if (Ci < 0) return -20;
    if (Cj < 0) return -21;
    if (batch < 0) return -23;
    if (batch == 0 || max_m == 0 || max_n == 0) return IRR_SUCCESS;
    if (!m) return -6;
    if (!n) return -7;
    if (!k) return -8;
    if (!A) return -10;
    if (!lda) return -13;
    if (!B) return -14;
    if (!ldb) return -17;
    if (!C) return -19;
    if (!ldc) return -22;
    int rc = check_device();
    if (rc) return rc;
    cudaStream_t s = (cudaStream_t)stream;
    int *tile_off = nullptr;
    if (work) {
        if (work_bytes < work_bytes_for(batch)) return IRR_ERR_WORKSPACE;
        tile_off = carve(work, batch).tile_off;
    }
    GemmArgs g{(int)ta, (int)tb, max_m, max_n, max_k, m, n, k, alpha, beta, A, Ai, Aj, lda, B, Bi, Bj, ldb,
               C, Ci, Cj, ldc, batch};
    launch_gemm_masked(g, nullptr, nullptr, tile_off, s, all_slots());
    return cudaGetLastError() == cudaSuccess ? IRR_SUCCESS : IRR_ERR_CUDA;
}

size_t irr_trsm_workspace_size(int batch) { return work_bytes_for(batch); }

int irr_trsm(irr_side_t side, irr_uplo_t uplo, irr_trans_t trans, irr_diag_t diag, int max_m, int max_n,
             const int *m, const int *n, double alpha, const double *const *T, int Ti, int Tj, const int *ldt,
             double *const *B, int Bi, int Bj, const int *ldb, int batch, void *work, size_t work_bytes,
             irr_stream_t stream) {
    if (side != IRR_LEFT && side != IRR_RIGHT) return -1;
    if (uplo != IRR_LOWER && uplo != IRR_UPPER) return -2;
    if (trans != IRR_NO_TRANS && trans != IRR_TRANS) return -3;
    if (diag != IRR_NON_UNIT && diag != IRR_UNIT) return -4;
    if (max_m < 0) return -5;
    if (max_n < 0) return -6;
    if (Ti < 0) return -11;
    if (Tj < 0) return -12;
    if (Bi < 0) return -15;
    if (Bj < 0) return -16;
    if (batch < 0) return -18;
    if (batch == 0 || max_m == 0 || max_n == 0) return IRR_SUCCESS;
    if (!m) return -7;
    if (!n) return -8;
    if (!T) return -10;
    if (!ldt) return -13;
    if (!B) return -14;
    if (!ldb) return -17;
    int rc = check_device();
    if (rc) return rc;
    cudaStream_t s = (cudaStream_t)stream;
    int *tile_off = nullptr, *counters = nullptr, *sort = nullptr;
    if (work) {
        if (work_bytes < work_bytes_for(batch)) return IRR_ERR_WORKSPACE;
        Work w = carve(work, batch);
        tile_off = w.tile_off;
        counters = w.counters;
        sort = w.sort;
        launch_size_sort(side == IRR_LEFT ? m : n, batch, sort, s);
    }
    TrsmArgs t{(int)side, (int)uplo, (int)trans, (int)diag, max_m, max_n, m, n, alpha, T, Ti, Tj, ldt,
               B, Bi, Bj, ldb, batch};
    run_trsm_masked(t, nullptr, counters, tile_off, s, sort);
    return cudaGetLastError() == cudaSuccess ? IRR_SUCCESS : IRR_ERR_CUDA;
}

int irr_laswp(int max_n, const int *n, double *const *A, int Ai, int Aj, const int *lda, int k1, int k2,
              const int *kcount, int *const *ipiv, int batch, irr_stream_t stream) {
    if (max_n < 0) return -1;
    if (Ai < 0) return -4;
    if (Aj < 0) return -5;
    if (k1 < 0) return -7;
    if (k2 < k1) return -8;
    if (batch < 0) return -11;
    if (batch == 0 || max_n == 0 || k2 == k1) return IRR_SUCCESS;
    if (!n) return -2;
    if (!A) return -3;
    if (!lda) return -6;
    if (!kcount) return -9;
    if (!ipiv) return -10;
    int rc = check_device();
    if (rc) return rc;
    launch_laswp_masked(max_n, n, A, Ai, Aj, lda, k1, k2, kcount, ipiv, batch, nullptr, (cudaStream_t)stream,
                        nullptr, all_slots());
    return cudaGetLastError() == cudaSuccess ? IRR_SUCCESS : IRR_ERR_CUDA;
}

}  // extern "C"

#!/usr/bin/env python
"""bench.py -- variable-size batched DGETRF (irrLU) on B200.

    python bench.py [--gpus N] [--steps K] [--warmup W] [--config C2] [--impl ours|reference]

A step is one irr_getrf (or irr_getrf_partial for the front configs) call on
the whole (per-rank) batch, i.e. every row of SURVEY §8(a), plus the NCCL
gather of the per-matrix status words when N > 1.  Inputs are restored from a
pristine device copy and L2 is flushed before every step, outside the timed
region; each step is timed with CUDA events on the launching stream; the
total over K steps is bracketed by a barrier + synchronize and reduced with
MAX over ranks.  Weak scaling: at N GPUs the global batch is N x the config's
batch, partitioned flop-balanced (LPT) over the ranks, each rank generating
only its own matrices (global-id-keyed values).

Metric (BASELINE.json): Gflop/s = sum FLOPS_DGETRF / time.
"""
from __future__ import annotations

import argparse
import json
import os
import statistics
import sys
import time

import numpy as np

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

import irrgen  # noqa: E402
from paper_conf_sc_abdelfattahgbtld22_b200 import flops as F  # noqa: E402
from paper_conf_sc_abdelfattahgbtld22_b200.shard import lpt_partition  # noqa: E402

METRIC = "variable-size batched DGETRF Gflop/s and % FP64/HBM roofline at 1/2/4/8 B200"
FP64_PEAK_TFLOPS = 148 * 64 * 2 * 1.965e9 / 1e12   # 37.2: 148 SM x 64 DFMA/clk x 2 x 1.965 GHz
FALLBACK_HBM_GBS = 6650.0


def peaks():
    p = os.path.join(ROOT, "MEASURED_PEAKS.json")
    try:
        with open(p) as f:
            d = json.load(f)
        return float(d["hbm_gbs"]), "measured"
    except Exception:
        return FALLBACK_HBM_GBS, "fallback"


# ------------------------------------------------------------------ clocks
class ClockSampler:
    """SM clock and throttle reasons sampled DURING the timed region: an NVML
    polling thread (every ~2 ms, so short timed regions still get samples);
    nvidia-smi is the fallback when NVML is not importable."""
    REASONS = (("hw_slowdown", "nvmlClocksEventReasonHwSlowdown"),
               ("hw_thermal_slowdown", "nvmlClocksEventReasonHwThermalSlowdown"),
               ("sw_thermal_slowdown", "nvmlClocksEventReasonSwThermalSlowdown"),
               ("sw_power_cap", "nvmlClocksEventReasonSwPowerCap"))

    def __init__(self, gpu_index: int):
        self.idx = gpu_index
        self.thread = None
        self.samples = []
        self.reasons = set()
        self.mx = 0.0

    def _run(self):
        import pynvml as nv
        h = self.h
        while not self.stop_flag:
            try:
                self.samples.append(float(nv.nvmlDeviceGetClockInfo(h, nv.NVML_CLOCK_SM)))
                bits = nv.nvmlDeviceGetCurrentClocksEventReasons(h)
                for name, attr in self.REASONS:
                    if bits & getattr(nv, attr, 0):
                        self.reasons.add(name)
            except Exception:
                pass
            time.sleep(0.002)

    def start(self):
        import threading
        try:
            import pynvml as nv
            nv.nvmlInit()
            # NVML enumerates all GPUs; map through CUDA_VISIBLE_DEVICES if set
            vis = os.environ.get("CUDA_VISIBLE_DEVICES")
            phys = self.idx
            if vis:
                toks = [t.strip() for t in vis.split(",") if t.strip()]
                if self.idx < len(toks) and toks[self.idx].isdigit():
                    phys = int(toks[self.idx])
            self.h = nv.nvmlDeviceGetHandleByIndex(phys)
            self.mx = float(nv.nvmlDeviceGetMaxClockInfo(self.h, nv.NVML_CLOCK_SM))
        except Exception:
            self.thread = None
            return
        self.stop_flag = False
        self.thread = threading.Thread(target=self._run, daemon=True)
        self.thread.start()

    def stop(self):
        if self.thread is None:
            return None
        self.stop_flag = True
        self.thread.join(timeout=5)
        if not self.samples:
            return None
        return {"sm_mhz": statistics.median(self.samples), "sm_max_mhz": self.mx,
                "reasons": sorted(self.reasons), "samples": len(self.samples), "source": "nvml"}


# ------------------------------------------------------------------ per-tier algorithmic work
def tier_of(m, n, tier_m_max=24576, l1=256):
    """0 = S (warp), 1 = M (CTA, in smem), 2 = L1 (CTA per matrix, m <= l1
    rows; 0 = off), 3 = L2 (grid-wide chain), -1 = empty; mirrors classify.cu."""
    m = np.asarray(m)
    n = np.asarray(n)
    lds = m | 1
    t = np.full(len(m), 3)
    if l1:
        t[m <= l1] = 2
    t[(lds * n) <= tier_m_max] = 1
    t[(m <= 32) & (n <= 32)] = 0
    t[(m == 0) | (n == 0)] = -1
    return t


def class_work(m, n, nb=32, tier_m_max=24576, l1=256, nbo=0):
    """Algorithmic (flops, bytes) per kernel class for one getrf step, SURVEY
    §8(d): flops = FLOPS_DGETRF of the matrices a class works on (the grid-wide
    tier's flops split by the step of the blocked algorithm each kernel
    performs: panel, U12 solve, trailing GEMM -- parts of FLOPS_DGETRF, no
    redundant work); bytes = each matrix read once and written once (16 m n +
    4 min(m,n) + 32), attributed to the tier that owns the matrix and, inside
    the grid-wide tier, to its kernel classes in proportion to their flops.
    Redundant traffic (the blocked algorithm re-streaming the trailing
    matrix) is never credited.  Tiers mirror classify.cu with the live tuning."""
    m = np.asarray(m, dtype=np.int64)
    n = np.asarray(n, dtype=np.int64)
    t = tier_of(m, n, tier_m_max, l1)
    out = {}
    for cls, tier in (("lu_small", 0), ("lu_mid", 1), ("lu_l1", 2)):
        sel = t == tier
        out[cls] = (float(F.getrf_flops(m[sel], n[sel]).sum()), float(F.getrf_bytes(m[sel], n[sel]).sum()))
    sel = t == 3
    mL, nL = m[sel], n[sel]
    tier_f = float(F.getrf_flops(mL, nL).sum())
    tier_b = float(F.getrf_bytes(mL, nL).sum())
    g_f = p_f = s_f = og_f = os_f = 0.0
    kL = np.minimum(mL, nL)
    two = nbo > nb
    for j in range(0, int(kL.max()) if len(kL) else 0, nb):
        act = kL > j
        if not act.any():
            break
        mm, nn, kk = mL[act], nL[act], kL[act]
        ib = np.minimum(nb, kk - j)
        # inner steps of the two-level tier stop at their outer block's edge
        ce = np.minimum(kk, (j // nbo + 1) * nbo) if two else nn
        Mr = np.maximum(mm - j - ib, 0).astype(np.float64)
        Nr = np.maximum(ce - j - ib, 0).astype(np.float64)
        g_f += float((2 * Mr * Nr * ib).sum())
        p_f += float(F.getrf_flops(mm - j, ib).sum())
        s_f += float((ib * ib * Nr).sum())
        if two and (j + nb) % nbo == 0 or (two and np.any(kk - j <= nb)):
            # end of an outer block [J, J + ibo) for the matrices whose block ends here
            J = (j // nbo) * nbo
            end = (kk <= j + nb) | ((j + nb) % nbo == 0)
            ibo = np.minimum(nbo, kk - J)[end].astype(np.float64)
            Mo = np.maximum(mm[end] - J - ibo, 0)
            No = np.maximum(nn[end] - J - ibo, 0)
            og_f += float((2 * Mo * No * ibo).sum())
            os_f += float((ibo * ibo * No).sum())
    share = (lambda f: tier_b * f / tier_f) if tier_f > 0 else (lambda f: 0.0)
    if two:
        out["gemm_trailing"] = (og_f, share(og_f))     # xgemm, K = nbo
        out["outer_trsm"] = (os_f, share(os_f))        # outer interchanges + U12 solve
    else:
        out["gemm_trailing"] = (g_f, share(g_f))
        out["swap_trsm"] = (s_f, share(s_f))
    out["panel"] = (p_f, share(p_f))
    out["strip"] = (g_f + s_f, share(g_f + s_f))  # fused interchange + TRSM + GEMM kernel (inner steps)
    out["grid_tier"] = (tier_f, tier_b)
    return out


def class_work_partial(n1, n2, nb=32, tier_m_max=24576, l1=256, nbo=0):
    """As class_work for F11, plus the partial-front steps a5.2 (2 n1^2 n2
    flops; F12 read + written, F11's factors read) and a5.3 (2 n1 n2^2 flops;
    F22 read + written, F21 and F12 read) with their read-once bytes."""
    n1 = np.asarray(n1, dtype=np.int64)
    n2 = np.asarray(n2, dtype=np.int64)
    out = class_work(n1, n1, nb, tier_m_max, l1, nbo)
    out["gemm_dcwi"] = (float((2.0 * n1 * n2 * n2).sum()), float((8.0 * (2 * n2 * n2 + n2 * n1 + n1 * n2)).sum()))
    out["trsm_leaf"] = (float((2.0 * n1 * n1 * n2).sum()), float((16.0 * n1 * n2 + 8.0 * n1 * n1).sum()))
    out["getrs"] = (float((2.0 * n1 * n1 * n2).sum()), float((16.0 * n1 * n2 + 8.0 * n1 * n1).sum()))
    return out


# ------------------------------------------------------------------ CPU oracle timing
def time_oracle(cfg, idx, target_s=10.0, threads=None):
    """Time the oracle (as it stands) on a bounded sample of the workload.
    Returns (gflops, cores, sample description, seconds)."""
    import oracle
    oracle.build()
    threads = threads or len(os.sched_getaffinity(0))
    rng = np.random.default_rng(12345)
    order = rng.permutation(idx)

    def run(sel):
        if cfg.kind == "getrf":
            mats = [irrgen.uniform_values(cfg.seed, int(g), int(cfg.m[g]), int(cfg.n[g])) for g in sel]
            fl = float(F.getrf_flops(cfg.m[sel], cfg.n[sel]).sum())
            t0 = time.perf_counter()
            oracle.getrf_batch(mats, nthreads=threads)
            return fl, time.perf_counter() - t0
        fronts = []
        for g in sel:
            a, b = int(cfg.m[g]), int(cfg.n[g])
            Fm = irrgen.front_values(cfg.seed, int(g), a + b)
            fronts.append(dict(F11=Fm[:a, :a].copy(order="F"), F12=Fm[:a, a:].copy(order="F"),
                               F21=Fm[a:, :a].copy(order="F"), F22=Fm[a:, a:].copy(order="F")))
        fl = float(F.partial_flops(cfg.m[sel], cfg.n[sel]).sum())
        t0 = time.perf_counter()
        oracle.getrf_partial_batch(fronts, nthreads=threads)
        return fl, time.perf_counter() - t0

    # calibrate on a small slice, then size the sample for ~target_s
    n0 = min(len(order), 64)
    fl0, t0 = run(order[:n0])
    rate = fl0 / max(t0, 1e-6)
    all_fl = F.getrf_flops(cfg.m[order], cfg.n[order]) if cfg.kind == "getrf" else \
        F.partial_flops(cfg.m[order], cfg.n[order])
    budget = rate * target_s
    cnt = int(np.searchsorted(np.cumsum(all_fl), budget)) + 1
    cnt = max(n0, min(len(order), cnt))
    sel = order[:cnt]
    fl, t = run(sel)
    desc = f"{cnt} of {len(idx)} matrices of {cfg.name} (uniform random sample, seed 12345), {fl:.3e} flop"
    return fl / t / 1e9, threads, desc, t


def cpu_model() -> str:
    try:
        with open("/proc/cpuinfo") as f:
            for line in f:
                if line.startswith("model name"):
                    return line.split(":", 1)[1].strip()
    except OSError:
        pass
    return "unknown"


# ------------------------------------------------------------------ reference arm
def run_reference(args, rank, world):
    """--impl reference: the CPU oracle (this tier's reference arm), rank 0 only."""
    if rank != 0:
        return
    cfg = irrgen.config(args.config)
    idx = np.arange(len(cfg.m))
    vals = []
    threads = len(os.sched_getaffinity(0))
    desc = ""
    for s in range(args.warmup + args.steps):
        g, cores, desc, secs = time_oracle(cfg, idx, target_s=args.ref_seconds, threads=threads)
        if s >= args.warmup:
            vals.append(g)
    v = float(np.mean(vals))
    line = {"impl": "reference", "metric": METRIC, "value": v, "unit": "Gflop/s", "n_gpus": world,
            "steps": args.steps, "warmup": args.warmup, "ms_per_step": None, "higher_is_better": True,
            "scaling": args.scaling, "vs_baseline": None, "dtype": "f64", "data": "synthetic",
            "config": {"workload": cfg.name, "description": cfg.description, "batch": int(len(cfg.m))},
            "cpu_baseline": {"value": v, "unit": "Gflop/s", "cores": threads, "kind": "oracle", "sample": desc,
                             "cpu_model": cpu_model()},
            "e2e": {"value": v, "unit": "Gflop/s", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}}
    print(json.dumps(line), flush=True)


# ------------------------------------------------------------------ our arm
def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=10)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--config", default="C5", choices=irrgen.CONFIG_NAMES,
                    help="workload (default C5: BASELINE.json's headline batch, the largest single-GPU config)")
    ap.add_argument("--scaling", default="strong", choices=["strong", "weak"],
                    help="strong: the config's batch split over the N ranks (T1 / TN, SURVEY §8(e)); "
                         "weak: N x the config")
    ap.add_argument("--impl", default="ours", choices=["ours", "reference"])
    ap.add_argument("--no-e2e", action="store_true")
    ap.add_argument("--e2e-chunks", type=int, default=8, help="chunks of the pipelined end-to-end call")
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--cpu-seconds", type=float, default=10.0)
    ap.add_argument("--ref-seconds", type=float, default=5.0)
    ap.add_argument("--profile-out", default=None, help="write per-kernel-class timings here (json)")
    ap.add_argument("--tune", action="append", default=[], help="key=value passed to irr_set_tuning (experiments)")
    args = ap.parse_args()

    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    if args.impl == "reference":
        run_reference(args, rank, world)
        return

    import torch
    import torch.distributed as dist
    from paper_conf_sc_abdelfattahgbtld22_b200 import irr
    from paper_conf_sc_abdelfattahgbtld22_b200.batch import FrontBatch, MatrixBatch

    # one process per GPU; IRR_BENCH_DIST_BACKEND=gloo is a test-only override
    # that lets several ranks share one GPU (exercises the N > 1 code path)
    backend = os.environ.get("IRR_BENCH_DIST_BACKEND", "nccl")
    dev_idx = local % max(1, torch.cuda.device_count())
    torch.cuda.set_device(dev_idx)
    dev = torch.device("cuda", dev_idx)
    for kv in args.tune:
        k, v = kv.split("=")
        irr.irr_set_tuning(k, int(v))
    if world > 1:
        if backend == "nccl":
            dist.init_process_group("nccl", device_id=dev)
        else:
            dist.init_process_group(backend)
    coll_dev = dev if backend == "nccl" else torch.device("cpu")

    # ---- workload: the config (strong) or world x the config (weak), LPT-sharded by flops
    cfg = irrgen.config(args.config, scale=float(world) if args.scaling == "weak" else 1.0)
    kind = cfg.kind
    work = F.getrf_flops(cfg.m, cfg.n) if kind == "getrf" else F.partial_flops(cfg.m, cfg.n)
    owner = lpt_partition(work, world)
    mine = np.nonzero(owner == rank)[0]
    m_loc, n_loc = cfg.m[mine], cfg.n[mine]
    flops_local = float(work[mine].sum())
    flops_global = float(work.sum())

    # C5 (200,000 fronts, 68 GB) is generated on the device, per rank, from
    # the same global-id-keyed stream (irrgen.device; byte-equal to the host
    # generator): neither a host copy nor a pristine device copy fits
    devgen = args.config.startswith("C5")
    host = None
    if kind == "getrf":
        B = MatrixBatch(m_loc, n_loc, device=dev)
        ld_loc = B.ld_h
        call = lambda: B.getrf()  # noqa: E731
        cw = class_work(m_loc, n_loc, irr.irr_get_tuning("nb"), irr.irr_get_tuning("tier_m_max"),
                        irr.irr_get_tuning("l1_rows") if irr.irr_get_tuning("l1") else 0,
                        irr.irr_get_tuning("nb_outer"))
        bytes_local = float(F.getrf_bytes(m_loc, n_loc).sum())
        gm, gn = m_loc, n_loc
    else:
        B = FrontBatch(m_loc, n_loc, device=dev)
        call = lambda: B.getrf_partial()  # noqa: E731
        cw = class_work_partial(m_loc, n_loc, irr.irr_get_tuning("nb"), irr.irr_get_tuning("tier_m_max"),
                                irr.irr_get_tuning("l1_rows") if irr.irr_get_tuning("l1") else 0,
                                irr.irr_get_tuning("nb_outer"))
        bytes_local = float(F.partial_bytes(m_loc, n_loc).sum())
        gm = gn = B.nf_h
    outs = [B.data, B.ipiv_data, B.info]
    if devgen:
        from irrgen import device as gdev
        filler = gdev.Filler(cfg.seed, gm, gn, B.ld_h, B.offsets, mine, dev)
        pristine = None
    else:
        host = torch.empty(B.total, dtype=torch.float64, pin_memory=True)
        hn = host.numpy()
        hn[:] = 0.0
        # values keyed by GLOBAL id so a matrix is identical at every N
        irrgen.fill_packed(cfg.seed, gm, gn, B.ld_h, B.offsets, hn, gids=mine)
        pristine = host.to(dev)
    flush = torch.empty(512 * 1024 * 1024, dtype=torch.uint8, device=dev)   # > 126 MB L2
    stream = torch.cuda.current_stream(dev)

    # status gather (the only collective, a6): per-matrix 8-byte status words
    # (info, FNV-1a of ipiv) from irr_status_words, padded to the largest shard
    pad = int(max(np.bincount(owner, minlength=world))) if world > 1 else len(mine)
    words = torch.zeros(2 * max(1, pad), dtype=torch.int32, device=dev)
    status = words if coll_dev == dev else torch.zeros_like(words, device=coll_dev)
    gathered = torch.zeros(world * 2 * max(1, pad), dtype=torch.int32, device=coll_dev) if world > 1 else None
    sm, sn = (B.m, B.n) if kind == "getrf" else (B.n1, B.n1)

    def step():
        call()
        if world > 1:
            irr.irr_status_words(B.batch, sm, sn, B.ipiv, B.info, words)
            if status is not words:
                status.copy_(words)
            dist.all_gather_into_tensor(gathered, status)

    def restore():
        if devgen:
            filler.fill(B.data)
        else:
            B.data.copy_(pristine)
        flush.zero_()

    # ---- warm-up
    for _ in range(args.warmup):
        restore()
        step()
    torch.cuda.synchronize()

    # ---- timed region
    irr.irr_profile_enable(100000)
    irr.irr_launch_count(reset=True)
    clocks = ClockSampler(dev_idx)
    if world > 1:
        dist.barrier()
    torch.cuda.synchronize()
    clocks.start()
    total_ms = 0.0
    evs = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)) for _ in range(args.steps)]
    for s in range(args.steps):
        restore()
        evs[s][0].record(stream)
        step()
        evs[s][1].record(stream)
    torch.cuda.synchronize()
    if world > 1:
        dist.barrier()
    torch.cuda.synchronize()
    clk = clocks.stop()
    step_ms = [a.elapsed_time(b) for a, b in evs]
    total_ms = float(sum(step_ms))
    launches = irr.irr_launch_count()
    try:  # per class, the union of its launch intervals (streams overlap)
        busy = irr.irr_profile_busy()
    except Exception:  # noqa: BLE001 -- fall back to the per-launch sums
        busy = None
    prof = irr.irr_profile_collect()
    irr.irr_profile_enable(0)
    if busy is not None:  # (sum of launch durations, launches) -> (busy time, launches)
        prof_busy = {k: (busy.get(k, v[0]), v[1]) for k, v in prof.items()}
    else:
        prof_busy = prof
    t = torch.tensor([total_ms], dtype=torch.float64, device=coll_dev)
    if world > 1:
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
    total_max_ms = float(t.item())
    ms_per_step = total_max_ms / args.steps
    value = flops_global / (ms_per_step * 1e-3) / 1e9

    # ---- parity spot-check on a few matrices of this rank (oracle-free: info must be >= 0)
    info_h = B.info[: B.batch].cpu().numpy()
    bad_info = int((info_h < 0).sum())

    # ---- e2e: host buffers through the public API, H2D + compute + D2H inside the timed region
    e2e = None
    if not args.no_e2e:
        e2e = run_e2e(args, B, kind, host, flush, stream, world, sm, sn, words, status, gathered, dist, irr,
                      work, mine, coll_dev)

    # ---- roofline of the dominant kernel class (rank-local, per step)
    hbm, hbm_src = peaks()
    # tiers S and M run on a forked stream concurrently with the large tiers:
    # their events also span the time spent waiting for SMs, so the dominant
    # kernel is taken among the main-stream classes whenever a large tier ran
    # With launches of one class on several streams (the grid tier's two
    # parts, tier S's second stream) the class time is the union of its
    # launch intervals, not their sum.
    side = {"lu_small", "lu_mid"}
    main = {k: v for k, v in prof_busy.items() if k not in side and v[1]}
    big_ran = any(k in main for k in ("lu_l1", "panel", "strip", "gemm_trailing"))
    cand = main if big_ran else {k: v for k, v in prof_busy.items() if v[1]}
    dom = max(cand.items(), key=lambda kv: kv[1][0])
    dname, (dms, dcnt) = dom
    # a class whose kernels run on two streams at once (tier S: the narrow
    # classes beside the wide ones) sums overlapping intervals: cap at the step
    dms_step = min(dms / args.steps, total_ms / args.steps)
    fl, by = cw.get(dname, (0.0, 0.0))
    t_f = fl / (FP64_PEAK_TFLOPS * 1e12)
    t_b = by / (hbm * 1e9)
    if t_b >= t_f:
        ach = by / (dms_step * 1e-3) / 1e9
        roof = {"bound": "hbm", "achieved": ach, "peak": hbm, "unit": "GB/s", "frac": ach / hbm}
    else:
        ach = fl / (dms_step * 1e-3) / 1e12
        # classes whose flops run on the FP64 tensor core (mma.sync DMMA) vs the DFMA pipe
        dmma = {"gemm_trailing", "strip", "lu_l1", "gemm_dcwi", "getrs", "outer_trsm"}
        roof = {"bound": "tensor" if dname in dmma else "alu", "achieved": ach, "peak": FP64_PEAK_TFLOPS,
                "unit": "TFLOP/s", "frac": ach / FP64_PEAK_TFLOPS}
    roof["kernel"] = dname
    roof["share_of_step"] = dms_step / (total_ms / args.steps)
    roof["launches_per_step"] = dcnt / args.steps
    roof["peak_source"] = ("measured: MEASURED_PEAKS.json hbm_gbs" if hbm_src == "measured" else
                           "fallback 6,650 GB/s (B200_PROFILING.md; MEASURED_PEAKS.json absent)") \
        if roof["bound"] == "hbm" else \
        ("measured FP64 tensor (DMMA m8n8k4) and DFMA rate 64 FMA/clk/SM (tools/microbench.cu, "
         "profiles/r01/microbench.txt) x 148 SM x 2 flop x 1.965 GHz = the FP64 nominal peak")
    roof["traffic"] = _ncu_traffic(args.config, dname, dcnt / args.steps)
    whole = {"flops": flops_local, "bytes": bytes_local,
             "fp64_frac": flops_local / (ms_per_step * 1e-3) / (FP64_PEAK_TFLOPS * 1e12),
             "hbm_frac": bytes_local / (ms_per_step * 1e-3) / (hbm * 1e9)}

    # ---- CPU baseline: the oracle on a bounded sample (rank 0, N = 1 only)
    cpu = None
    if rank == 0 and world == 1 and not args.no_cpu_baseline:
        g, cores, desc, secs = time_oracle(irrgen.config(args.config), np.arange(len(cfg.m)),
                                           target_s=args.cpu_seconds)
        cpu = {"value": g, "unit": "Gflop/s", "cores": cores, "kind": "oracle", "sample": desc,
               "seconds": secs, "cpu_model": cpu_model()}

    if args.profile_out and rank == 0:
        with open(args.profile_out, "w") as f:
            json.dump({k: {"ms_per_step": v[0] / args.steps, "launches_per_step": v[1] / args.steps,
                           "alg_flops": cw.get(k, (0, 0))[0], "alg_bytes": cw.get(k, (0, 0))[1]}
                       for k, v in prof.items() if v[1]}, f, indent=1)

    if rank == 0:
        line = {"metric": METRIC, "value": value, "unit": "Gflop/s", "n_gpus": world, "steps": args.steps,
                "warmup": args.warmup, "ms_per_step": ms_per_step, "higher_is_better": True,
                "scaling": args.scaling, "vs_baseline": None, "dtype": "f64",
                "data": "synthetic (seeded splitmix64 values U[-1,1), sizes per BASELINE config)",
                "config": {"workload": cfg.name if (world == 1 or args.scaling == "strong") else f"{world}x{args.config}",
                           "description": irrgen.config(args.config).description,
                           "batch_per_gpu": int(B.batch), "global_batch": int(len(cfg.m)),
                           "sharding": "LPT by flops" if world > 1 else "none",
                           "l2": "flushed (512 MB write) and inputs restored before every step, untimed",
                           "inputs": "generated on the device per step (untimed)" if devgen else
                                     "restored from a pristine device copy per step (untimed)",
                           "tuning": {k: irr.irr_get_tuning(k) for k in ("nb", "tier_m_max", "panel_rows")}},
                "gpu_launches": int(launches), "roofline": roof, "whole_step": whole,
                "kernel_ms_per_step": {k: v[0] / args.steps for k, v in prof.items() if v[1]},
                "kernel_busy_ms_per_step": {k: v[0] / args.steps for k, v in prof_busy.items() if v[1]},
                "clocks": clk, "e2e": e2e, "cpu_baseline": cpu, "info_negative": bad_info}
        print(json.dumps(line), flush=True)
    if world > 1:
        dist.destroy_process_group()


def run_e2e(args, B, kind, host, flush, stream, world, sm, sn, words, status, gathered, dist, irr, work, mine,
            coll_dev):
    """The metric end to end through the public entry points getrf_host /
    getrf_partial_host: every step copies the inputs from pinned host memory,
    factors them and copies factors, pivots and info back, chunk-pipelined
    (H2D of chunk c+1 / compute of chunk c / D2H of chunk c-1 overlap).  For
    the device-generated C5 the host buffers are filled once (untimed) by a
    device-to-host copy; when two host copies of the batch do not fit in RAM,
    the largest prefix of the batch that does is timed and named."""
    import psutil
    import torch
    from paper_conf_sc_abdelfattahgbtld22_b200.batch import (FrontBatch, MatrixBatch, getrf_host,
                                                             getrf_partial_host)
    Be, note = B, "whole batch"
    if host is None:
        avail = psutil.virtual_memory().available
        budget = int(avail * 0.50) // 16          # doubles per host copy (two pinned copies: in, out)
        i1 = B.batch
        if B.total > budget:
            ends = B.offsets + (B.ld_h * (B.n_h if kind == "getrf" else B.nf_h))
            i1 = int(np.searchsorted(ends, budget, side="right"))
            note = (f"prefix of {i1} of {B.batch} matrices ({ends[i1 - 1] * 8 / 1e9:.1f} GB): two pinned copies of "
                    f"the whole batch ({B.total * 16 / 1e9:.0f} GB) exceed the host's available RAM "
                    f"({avail / 1e9:.0f} GB)")
        if i1 < B.batch:
            if kind == "getrf":
                Be = MatrixBatch(B.m_h[:i1], B.n_h[:i1], data=B.data)
            else:
                raise RuntimeError("partial e2e prefix not supported")
        host = torch.empty(Be.total, dtype=torch.float64, pin_memory=True)
        host.copy_(B.data[: Be.total])          # the device-generated inputs, once (untimed)
        sel = mine[: Be.batch]
    else:
        sel = mine
    outs = [Be.data, Be.ipiv_data, Be.info]
    res_host = [torch.empty(o.numel(), dtype=o.dtype, pin_memory=True) for o in outs]
    h2d = host.numel() * 8
    d2h = sum(o.numel() * o.element_size() for o in outs)
    flops = float(work[sel].sum())
    e2e_fn = getrf_host if kind == "getrf" else getrf_partial_host
    pipe = None
    e_ms = []
    for s in range(args.warmup + args.steps):
        flush.zero_()
        torch.cuda.synchronize()
        if world > 1:
            dist.barrier()
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        a.record(stream)
        pipe = e2e_fn(Be, host, res_host[0], res_host[1], res_host[2], chunks=args.e2e_chunks, pipe=pipe)
        if world > 1:
            irr.irr_status_words(Be.batch, sm, sn, Be.ipiv, Be.info, words)
            if status is not words:
                status.copy_(words)
            dist.all_gather_into_tensor(gathered, status)
        b.record(stream)
        torch.cuda.synchronize()
        if s >= args.warmup:
            e_ms.append(a.elapsed_time(b))
    te = torch.tensor([float(np.sum(e_ms))], dtype=torch.float64, device=coll_dev)
    if world > 1:
        ft = torch.tensor([flops], dtype=torch.float64, device=te.device)
        dist.all_reduce(te, op=dist.ReduceOp.MAX)
        dist.all_reduce(ft, op=dist.ReduceOp.SUM)
        flops = float(ft.item())
    e_step = float(te.item()) / args.steps
    return {"value": flops / (e_step * 1e-3) / 1e9, "unit": "Gflop/s", "ms_per_step": e_step,
            "h2d_bytes_per_step": int(h2d), "d2h_bytes_per_step": int(d2h), "batch": note,
            "pipeline": f"{args.e2e_chunks} chunks: H2D / getrf / D2H overlapped (pinned host buffers)"}


def _ncu_traffic(config, kname, launches_per_step):
    """dram bytes per launch of `kname` from a committed ncu --set full summary, else None."""
    p = os.path.join(ROOT, "profiles", f"ncu_traffic_{config}.json")
    try:
        with open(p) as f:
            d = json.load(f)
        return d.get(kname)
    except Exception:
        return None


if __name__ == "__main__":
    main()

"""Measure the §8(f) NEXT rows on B200: each line is one JSON
object with the algorithmic work, the CUDA-event time (mean of --reps after
warm-up, inputs restored between runs, untimed) and the roofline fraction
(FP64 37.2 TFLOP/s; HBM = MEASURED_PEAKS.json).

  zgetrf     irr_zgetrf on complex batches shaped like C2 (10,000, dims U{1..256})
             and C3 (2,000 square U{256..1024}); flops = 6 FMULS + 2 FADDS of
             LAPACK's zgetrf count (Q1's complex analogue).
  lapack     irr_getrf_partial_lapack vs irr_getrf_partial on C4-shaped fronts
             (a bounded sample: --c4-scale).
  tree       AssemblyTree.factor() on a depth --depth nested-dissection tree:
             partial flops (Q2) of every front + extend-add bytes per level.
  large      single matrices / small batches of 2048-8192 (the few-large
             regime, Fig. 11): irr_getrf, and the cuSOLVER getrf behind
             torch.linalg.lu_factor on the same matrix as context only.

    python tools/bench_next.py [--what zgetrf,lapack,tree,large] [--reps 5]
"""
import argparse
import json
import os
import sys

import numpy as np
import torch

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import irrgen  # noqa: E402
from paper_conf_sc_abdelfattahgbtld22_b200 import flops as F  # noqa: E402
from paper_conf_sc_abdelfattahgbtld22_b200 import irr  # noqa: E402
from paper_conf_sc_abdelfattahgbtld22_b200.batch import FrontBatch, MatrixBatch, ZMatrixBatch  # noqa: E402

FP64 = 148 * 64 * 2 * 1.965e9
HBM = json.load(open(os.path.join(ROOT, "MEASURED_PEAKS.json")))["hbm_gbs"] * 1e9 \
    if os.path.exists(os.path.join(ROOT, "MEASURED_PEAKS.json")) else 6.65e12


def timed(restore, call, reps):
    s = torch.cuda.current_stream()
    for _ in range(2):
        restore()
        call()
    torch.cuda.synchronize()
    ts = []
    for _ in range(reps):
        restore()
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        a.record(s)
        call()
        b.record(s)
        torch.cuda.synchronize()
        ts.append(a.elapsed_time(b))
    return float(np.mean(ts))


def zflops(m, n):
    m = np.asarray(m, dtype=np.float64)
    n = np.asarray(n, dtype=np.float64)
    big, k = np.maximum(m, n), np.minimum(m, n)
    fmuls = 0.5 * big * k * k - k ** 3 / 6 + big * k / 2 - k * k / 2 + 2 * k / 3
    fadds = 0.5 * big * k * k - k ** 3 / 6 - big * k / 2 + k / 6
    return np.where(k > 0, 6 * fmuls + 2 * fadds, 0.0)


def out(d):
    print(json.dumps(d), flush=True)


def bench_zgetrf(reps):
    for name in ("C2", "C3"):
        cfg = irrgen.config(name)
        B = ZMatrixBatch(cfg.m, cfg.n)
        torch.manual_seed(1)
        pristine = torch.rand(B.total, dtype=torch.float64, device="cuda") * 2 - 1
        ms = timed(lambda: B.data.copy_(pristine), lambda: B.getrf(), reps)
        fl = float(zflops(cfg.m, cfg.n).sum())
        by = float((32.0 * cfg.m * cfg.n + 4 * np.minimum(cfg.m, cfg.n) + 32).sum())
        out({"what": "zgetrf", "workload": f"{name}-shaped complex", "batch": B.batch, "ms": ms,
             "gflops": fl / ms / 1e6, "fp64_frac": fl / (ms * 1e-3) / FP64, "hbm_frac": by / (ms * 1e-3) / HBM})


def bench_lapack(reps, scale):
    cfg = irrgen.config("C4", scale=scale)
    Fb = FrontBatch(cfg.m, cfg.n)
    host = np.zeros(Fb.total)
    irrgen.fill_packed(cfg.seed, Fb.nf_h, Fb.nf_h, Fb.ld_h, Fb.offsets, host)
    pristine = torch.from_numpy(host).cuda()
    fl = float(F.partial_flops(cfg.m, cfg.n).sum())
    for lapack in (False, True):
        ms = timed(lambda: Fb.data.copy_(pristine), lambda: Fb.getrf_partial(lapack=lapack), reps)
        out({"what": "partial_lapack" if lapack else "partial", "workload": f"C4 x {scale}", "batch": Fb.batch,
             "ms": ms, "gflops": fl / ms / 1e6, "fp64_frac": fl / (ms * 1e-3) / FP64})


def bench_tree(reps, depth):
    from paper_conf_sc_abdelfattahgbtld22_b200.tree import AssemblyTree
    tree = irrgen.assembly_tree(5, depth, s0=12.0, growth=1.5)
    T = AssemblyTree(tree.n1, tree.n2, tree.parent, tree.rel, tree.levels)
    torch.manual_seed(2)
    pristine = torch.rand(T.F.total, dtype=torch.float64, device="cuda") * 2 - 1
    ms = timed(lambda: T.F.data.copy_(pristine), lambda: T.factor(), reps)
    fl = float(F.partial_flops(tree.n1, tree.n2).sum())
    out({"what": "tree", "depth": depth, "fronts": int(len(tree.n1)), "max_front": int(tree.nf.max()), "ms": ms,
         "gflops": fl / ms / 1e6, "fp64_frac": fl / (ms * 1e-3) / FP64,
         "levels": len(tree.levels)})


def bench_large(reps):
    for n, cnt in ((2048, 1), (4096, 1), (6144, 1), (8192, 1), (4096, 8)):
        B = MatrixBatch([n] * cnt, [n] * cnt)
        torch.manual_seed(3)
        pristine = torch.rand(B.total, dtype=torch.float64, device="cuda") * 2 - 1
        fl = float(F.getrf_flops([n] * cnt, [n] * cnt).sum())
        res = {}
        for nbo, split in ((0, 0), (128, 0), (128, 1)):
            irr.irr_reset_tuning()
            irr.irr_set_tuning("nb_outer", nbo)
            irr.irr_set_tuning("split_strip", split)
            ms = timed(lambda: B.data.copy_(pristine), lambda: B.getrf(), reps)
            res[f"nb_outer={nbo}" + (",split_strip=1" if split else "")] = {"ms": ms, "gflops": fl / ms / 1e6}
        irr.irr_reset_tuning()
        A = pristine[: n * n].view(n, n).clone()
        ms_ref = timed(lambda: None, lambda: torch.linalg.lu_factor(A), reps) * cnt
        out({"what": "large", "n": n, "count": cnt, "irr": res,
             "cusolver_via_torch_context": {"ms": ms_ref, "gflops": fl / ms_ref / 1e6}})


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--what", default="zgetrf,lapack,tree,large")
    ap.add_argument("--reps", type=int, default=5)
    ap.add_argument("--c4-scale", type=float, default=0.2)
    ap.add_argument("--depth", type=int, default=14)
    ap.add_argument("--tune", action="append", default=[])
    a = ap.parse_args()
    for kv in a.tune:
        k, v = kv.split("=")
        irr.irr_set_tuning(k, int(v))
    w = a.what.split(",")
    if "zgetrf" in w:
        bench_zgetrf(a.reps)
    if "lapack" in w:
        bench_lapack(a.reps, a.c4_scale)
    if "tree" in w:
        bench_tree(a.reps, a.depth)
    if "large" in w:
        bench_large(a.reps)


if __name__ == "__main__":
    main()

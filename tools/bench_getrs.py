"""Measure irr_getrs (X <- U^-1 L^-1 P^T B with the
getrf factors) on a C2-like batch of square systems.

Batch: `--batch` matrices, n ~ U{1..n_max} (seeded), factored once by
irr_getrf (untimed); then `--reps` solves timed with CUDA events on the
launching stream after warm-up.  nrhs = `--nrhs` (0 = nrhs_i = n_i, the
square right-hand sides of a5.2).  Values are torch randn (timing only;
parity is tests/test_gpu_getrs.py).

Algorithmic work per system: 2 n^2 nrhs flops; bytes 8 n^2 (read L\\U) +
16 n nrhs (B read + written) + 4 n (ipiv).  Both fractions are printed
(FP64 peak 37.2 TFLOP/s as in DESIGN §5, HBM = MEASURED_PEAKS.json).

    python tools/bench_getrs.py [--batch 10000] [--n-max 256] [--nrhs 0|k] [--reps 20]
"""
import argparse
import json
import os
import sys

import numpy as np
import torch

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
from paper_conf_sc_abdelfattahgbtld22_b200.batch import MatrixBatch  # noqa: E402

FP64_PEAK = 148 * 64 * 2 * 1.965e9


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--batch", type=int, default=10000)
    ap.add_argument("--n-max", type=int, default=256)
    ap.add_argument("--nrhs", type=int, default=0)
    ap.add_argument("--reps", type=int, default=20)
    ap.add_argument("--seed", type=int, default=3)
    ap.add_argument("--tune", action="append", default=[], help="irr_set_tuning key=value")
    a = ap.parse_args()
    from paper_conf_sc_abdelfattahgbtld22_b200 import irr
    for kv in a.tune:
        k, v = kv.split("=")
        irr.irr_set_tuning(k, int(v))
    rng = np.random.default_rng(a.seed)
    n = rng.integers(1, a.n_max + 1, size=a.batch)
    nrhs = n if a.nrhs == 0 else np.full(a.batch, a.nrhs)
    A = MatrixBatch(n, n)
    Bm = MatrixBatch(n, nrhs, with_ipiv=False)
    torch.manual_seed(a.seed)
    A.data.copy_(torch.randn(A.total, dtype=torch.float64, device="cuda"))
    Bm.data.copy_(torch.randn(Bm.total, dtype=torch.float64, device="cuda"))
    A.getrf()
    torch.cuda.synchronize()
    s = torch.cuda.current_stream()
    for _ in range(3):
        A.getrs(Bm, stream=s)
    torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record(s)
    for _ in range(a.reps):
        A.getrs(Bm, stream=s)
    e1.record(s)
    torch.cuda.synchronize()
    ms = e0.elapsed_time(e1) / a.reps
    n64, r64 = n.astype(np.float64), nrhs.astype(np.float64)
    flops = float((2 * n64 * n64 * r64).sum())
    byts = float((8 * n64 * n64 + 16 * n64 * r64 + 4 * n64).sum())
    peak = json.load(open(os.path.join(ROOT, "MEASURED_PEAKS.json")))["hbm_gbs"]
    gf = flops / (ms * 1e-3) / 1e9
    gbs = byts / (ms * 1e-3) / 1e9
    print(json.dumps({"kernel": "getrs", "batch": a.batch, "n_max": a.n_max, "nrhs": a.nrhs or "n_i", "tune": a.tune,
                      "ms_per_solve": round(ms, 4), "gflops": round(gf, 1), "fp64_frac": round(gf * 1e9 / FP64_PEAK, 3),
                      "achieved_gbs": round(gbs, 1), "hbm_frac": round(gbs / peak, 3), "alg_flops": flops,
                      "alg_bytes": byts}))


if __name__ == "__main__":
    main()

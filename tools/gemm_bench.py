"""irr_gemm throughput on uniform batches (GEMM-core efficiency check).

    python tools/gemm_bench.py [--m 2048 --n 2048 --k 1024 --batch 16]
"""
import argparse
import os
import sys

import numpy as np
import torch

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
from paper_conf_sc_abdelfattahgbtld22_b200 import irr  # noqa: E402
from paper_conf_sc_abdelfattahgbtld22_b200.batch import MatrixBatch  # noqa: E402

ap = argparse.ArgumentParser()
ap.add_argument("--m", type=int, default=2048)
ap.add_argument("--n", type=int, default=2048)
ap.add_argument("--k", type=int, default=1024)
ap.add_argument("--batch", type=int, default=16)
ap.add_argument("--reps", type=int, default=5)
ap.add_argument("--tune", action="append", default=[])
ap.add_argument("--ta", type=int, default=0)
ap.add_argument("--tb", type=int, default=0)
a = ap.parse_args()
for kv in a.tune:
    kk, vv = kv.split("=")
    irr.irr_set_tuning(kk, int(vv))
b = a.batch
A = MatrixBatch([a.m] * b, [a.k] * b, with_ipiv=False)
B = MatrixBatch([a.k] * b, [a.n] * b, with_ipiv=False)
Cm = MatrixBatch([a.m] * b, [a.n] * b, with_ipiv=False)
for X in (A, B, Cm):
    X.data.copy_(torch.rand(X.total, dtype=torch.float64))


def i32(v):
    return torch.full((b,), v, dtype=torch.int32, device="cuda")


work = torch.empty(irr.irr_gemm_workspace_size(b), dtype=torch.uint8, device="cuda")
args = (0, 0, a.m, a.n, a.k, i32(a.m), i32(a.n), i32(a.k), -1.0, A.ptr, 0, 0, A.ld, B.ptr, 0, 0, B.ld, 1.0,
        Cm.ptr, 0, 0, Cm.ld, b)
irr.irr_gemm(*args, work=work)
torch.cuda.synchronize()
ts = []
for _ in range(a.reps):
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record()
    irr.irr_gemm(*args, work=work)
    e1.record()
    torch.cuda.synchronize()
    ts.append(e0.elapsed_time(e1))
t = min(ts)
fl = 2.0 * a.m * a.n * a.k * b
print(f"irr_gemm {b} x {a.m}x{a.n}x{a.k}: {t:.3f} ms  {fl / t / 1e9:.1f} GFLOP/s "
      f"({100 * fl / t / 1e9 / 37200:.1f}% of 37.2 TF)")
# check one product against torch (fp64)
i = 0
Ah = A.data[A.offsets[i]:A.offsets[i] + a.m * a.k].view(a.k, a.m).T
Bh = B.data[B.offsets[i]:B.offsets[i] + a.k * a.n].view(a.n, a.k).T

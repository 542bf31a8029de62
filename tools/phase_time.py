"""Per-phase SM-cycle breakdown of the CTA-per-matrix kernels (tuning
phase_timing=1; thread 0 of every CTA accumulates clock64 deltas).

    python tools/phase_time.py --config C2
"""
import argparse
import os
import sys

import numpy as np
import torch

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import irrgen  # noqa: E402
from paper_conf_sc_abdelfattahgbtld22_b200 import irr  # noqa: E402
from paper_conf_sc_abdelfattahgbtld22_b200.batch import MatrixBatch  # noqa: E402

NAMES = ["L1 panel wb / (M: -)", "L1 swap plan", "L1 gemm", "L1 stage | M load", "L1 panel | M panel",
         "L1 gather | M trsm", "L1 trsm | M gemm", "L1 scatter | M store"]

ap = argparse.ArgumentParser()
ap.add_argument("--config", default="C2")
ap.add_argument("--scale", type=float, default=1.0)
ap.add_argument("--tune", action="append", default=[])
a = ap.parse_args()
for kv in a.tune:
    k, v = kv.split("=")
    irr.irr_set_tuning(k, int(v))
cfg = irrgen.config(a.config, scale=a.scale)
B = MatrixBatch(cfg.m, cfg.n)
host = np.zeros(B.total)
irrgen.fill_packed(cfg.seed, cfg.m, cfg.n, B.ld_h, B.offsets, host)
B.data.copy_(torch.from_numpy(host))
B.getrf()
torch.cuda.synchronize()
B.data.copy_(torch.from_numpy(host))
irr.irr_set_tuning("phase_timing", 1)
B.getrf()
torch.cuda.synchronize()
w = B.work[128:128 + 64].cpu().numpy().view(np.uint64)
tot = float(w.sum()) or 1.0
for nm, v in zip(NAMES, w):
    print(f"{nm:14s} {float(v):.3e} cycles  {100 * float(v) / tot:5.1f}%")
big = ~((cfg.m <= 32) & (cfg.n <= 32))
ksum = float(np.minimum(cfg.m, cfg.n)[big].sum())
print(f"non-S column steps {ksum:.3e}; per step: slot3 {float(w[3]) / ksum:.0f}, slot4 {float(w[4]) / ksum:.0f}, "
      f"slot1 {float(w[1]) / ksum:.0f}, slot2 {float(w[2]) / ksum:.0f} cycles")

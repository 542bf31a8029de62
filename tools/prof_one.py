"""Run irr_getrf / irr_getrf_partial on one config a few times (for ncu).

    python tools/prof_one.py --config C2 [--scale 1.0] [--reps 2]
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
from paper_conf_sc_abdelfattahgbtld22_b200.batch import FrontBatch, MatrixBatch  # noqa: E402

ap = argparse.ArgumentParser()
ap.add_argument("--config", default="C2")
ap.add_argument("--scale", type=float, default=1.0)
ap.add_argument("--reps", type=int, default=2)
ap.add_argument("--tune", action="append", default=[], help="key=value for irr_set_tuning")
a = ap.parse_args()
for kv in a.tune:
    k, v = kv.split("=")
    irr.irr_set_tuning(k, int(v))
cfg = irrgen.config(a.config, scale=a.scale)
if cfg.kind == "getrf":
    B = MatrixBatch(cfg.m, cfg.n)
    host = np.zeros(B.total)
    irrgen.fill_packed(cfg.seed, cfg.m, cfg.n, B.ld_h, B.offsets, host)
    call = B.getrf
else:
    B = FrontBatch(cfg.m, cfg.n)
    host = np.zeros(B.total)
    irrgen.fill_packed(cfg.seed, B.nf_h, B.nf_h, B.ld_h, B.offsets, host)
    call = B.getrf_partial
pristine = torch.from_numpy(host).cuda()
for r in range(a.reps):
    B.data.copy_(pristine)
    call()
torch.cuda.synchronize()
print("done", a.config, B.batch, "info<0:", int((B.info[:B.batch] < 0).sum()))

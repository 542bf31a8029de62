"""Measure irr_extend_add on one synthetic tree
level against the HBM roofline.

Level: P parents with np ~ U[1, np_max], each with `kids` children whose
Schur complement order is U[0.25, 0.75] * np, rel a sorted random subset (the
recipe of irrgen.extend_add_level; values drawn on the device with torch,
since only timing is measured here -- parity is tests/test_gpu_extend_add.py).
Sibling rounds (one call per child index) as a tree traversal would issue.

Algorithmic bytes per child element: 8 (read F22) + 16 (read + write the
parent entry) + rel reads (4 * n2 per child, negligible).  The parent fronts
(GBs) are far larger than L2, and each round touches a different random subset.
Timed with CUDA events on the launching stream, warm-up first.

    python tools/bench_extend_add.py [--parents 512] [--np-max 2048] [--kids 2] [--reps 10]
"""
import argparse
import json
import os
import sys

import numpy as np
import torch

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
from paper_conf_sc_abdelfattahgbtld22_b200 import irr  # noqa: E402


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--parents", type=int, default=512)
    ap.add_argument("--np-max", type=int, default=2048)
    ap.add_argument("--kids", type=int, default=2)
    ap.add_argument("--reps", type=int, default=10)
    ap.add_argument("--seed", type=int, default=1)
    a = ap.parse_args()
    rng = np.random.default_rng(a.seed)
    dev = "cuda"
    nps = rng.integers(1, a.np_max + 1, size=a.parents)
    Pt = [torch.randn(int(s), int(s), dtype=torch.float64, device=dev) for s in nps]
    rounds = []
    elems = 0
    for r in range(a.kids):
        n2, Ct, rel = [], [], []
        for p, s in enumerate(nps):
            s = int(s)
            k = int(rng.integers(max(1, s // 4), max(1, (3 * s) // 4) + 1))
            k = min(max(k, 1), s)
            n2.append(k)
            Ct.append(torch.randn(k, k, dtype=torch.float64, device=dev))
            rel.append(torch.from_numpy(np.sort(rng.choice(s, size=k, replace=False)).astype(np.int32)).to(dev))
            elems += k * k
        i32 = lambda x: torch.tensor(x, dtype=torch.int32, device=dev)  # noqa: E731
        rounds.append(dict(
            batch=a.parents, max_n2=max(n2), n2=i32(n2),
            F22=torch.tensor([t.data_ptr() for t in Ct], dtype=torch.int64, device=dev),
            ld22=i32(n2), rel=torch.tensor([t.data_ptr() for t in rel], dtype=torch.int64, device=dev),
            np_=i32([int(s) for s in nps]),
            Fp=torch.tensor([t.data_ptr() for t in Pt], dtype=torch.int64, device=dev),
            ldp=i32([int(s) for s in nps]), info=torch.empty(a.parents, dtype=torch.int32, device=dev),
            keep=(Ct, rel)))
    s = torch.cuda.current_stream()

    def level():
        for R in rounds:
            irr.irr_extend_add(R["batch"], R["max_n2"], R["n2"], R["F22"], R["ld22"], R["rel"], R["np_"],
                               R["Fp"], R["ldp"], R["info"], stream=s)

    for _ in range(3):
        level()
    torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record(s)
    for _ in range(a.reps):
        level()
    e1.record(s)
    torch.cuda.synchronize()
    ms = e0.elapsed_time(e1) / a.reps
    alg = elems * 24 + sum(int(R["n2"].sum()) for R in rounds) * 4
    peak = json.load(open(os.path.join(ROOT, "MEASURED_PEAKS.json")))["hbm_gbs"]
    gbs = alg / (ms * 1e-3) / 1e9
    assert all(int(R["info"].abs().sum()) == 0 for R in rounds)
    print(json.dumps({"kernel": "extend_add", "parents": a.parents, "np_max": a.np_max, "kids": a.kids,
                      "child_elements": elems, "ms_per_level": round(ms, 4), "alg_bytes": alg,
                      "achieved_gbs": round(gbs, 1), "peak_gbs": peak, "frac": round(gbs / peak, 3),
                      "launches_per_level": a.kids}))


if __name__ == "__main__":
    main()

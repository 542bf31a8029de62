"""Parity on EVERY matrix of the BASELINE.json configs (C1, C1-big, C2, C3, C4)
and on a stated sample of C5 (64 of its ~2,000 fronts >= 1024 and 2,000 of
the rest; every front >= 1024 with IRR_PARITY_C5_ALL=1),
through the C ABI in the launch configuration bench.py times (the whole
config as one irr_getrf / irr_getrf_partial call, ld = m, 256-B aligned).

The oracle side runs batched in C (oracle/check.c: oracle_getrf /
oracle_getrf_partial on copies of the regenerated originals, OpenMP over
matrices); the rules are tests/parity.py (north_star tolerances, SURVEY §8(c)
Q11-Q13, G8 |l| <= 1).  PAPER.md L106 (§III-B) defines the result checked:
P L U = A.  Counts per config are printed (pytest -s) and asserted.

Marked `full` as well as `gpu`: the round-end `pytest -m gpu` runs them
(several minutes of oracle time on the box's host cores).
"""
import os
import time

import numpy as np
import pytest

import irrgen
import oracle

pytestmark = [pytest.mark.gpu, pytest.mark.full]

torch = pytest.importorskip("torch")
if not torch.cuda.is_available():
    pytest.skip("no CUDA device", allow_module_level=True)

from parity import assess_getrf, assess_partial  # noqa: E402
from paper_conf_sc_abdelfattahgbtld22_b200 import irr  # noqa: E402
from paper_conf_sc_abdelfattahgbtld22_b200.batch import FrontBatch, MatrixBatch  # noqa: E402

CHUNK = 1 << 30   # doubles of host buffer per checked chunk (8 GiB: the 47 C4 fronts >= 3072
                  # fall in one chunk, so the big oracle runs spread over every thread)
THREADS = len(os.sched_getaffinity(0))


@pytest.fixture(autouse=True)
def _reset_tuning():
    irr.irr_reset_tuning()
    yield
    irr.irr_reset_tuning()


def _merge(tot, st):
    for k, v in st.items():
        if k.startswith("max_"):
            tot[k] = max(tot.get(k, 0.0), v)
        else:
            tot[k] = tot.get(k, 0) + v


def _groups(sizes, sel):
    """Split the selected matrices into groups of <= CHUNK elements."""
    out, cur, acc = [], [], 0
    for i in sel:
        s = int(sizes[i]) + 32
        if cur and acc + s > CHUNK:
            out.append(cur)
            cur, acc = [], 0
        cur.append(i)
        acc += s
    if cur:
        out.append(cur)
    return out


def _gather(B, idx, kdim):
    """Host copies of the selected matrices / pivots in a local packed layout."""
    idx = np.asarray(idx)
    ld, n = B.ld_h[idx], (B.n_h[idx] if kdim == "getrf" else B.nf_h[idx])
    off, total = irrgen.packed_offsets(ld, n)
    res = np.zeros(total)
    k = B.k_h[idx] if kdim == "getrf" else B.n1_h[idx]
    ioff, itotal = irrgen.packed_offsets(np.ones_like(k), np.maximum(k, 1))
    ip = np.zeros(itotal, dtype=np.int32)
    # contiguous runs of the batch are copied in one piece
    runs = np.split(np.arange(len(idx)), np.nonzero(np.diff(idx) != 1)[0] + 1)
    for r in runs:
        a, b = int(idx[r[0]]), int(idx[r[-1]])
        e0 = int(B.offsets[a])
        e1 = int(B.offsets[b] + B.ld_h[b] * (B.n_h[b] if kdim == "getrf" else B.nf_h[b]))
        src = B.data[e0:e1].cpu().numpy()
        for q in r:
            i = int(idx[q])
            s0 = int(B.offsets[i]) - e0
            cnt = int(B.ld_h[i] * n[q])
            res[off[q]: off[q] + cnt] = src[s0: s0 + cnt]
        p0 = int(B.ipiv_off[a])
        p1 = int(B.ipiv_off[b] + max(1, k[r[-1]]))
        psrc = B.ipiv_data[p0:p1].cpu().numpy()
        for q in r:
            i = int(idx[q])
            ip[ioff[q]: ioff[q] + k[q]] = psrc[int(B.ipiv_off[i]) - p0: int(B.ipiv_off[i]) - p0 + k[q]]
    return ld, n, off, res, ioff, ip


def _check_getrf_batch(B, seed, gids, sel, label):
    info = B.info.cpu().numpy()[: B.batch]
    tot = {}
    sizes = B.ld_h * B.n_h
    for grp in _groups(sizes, sel):
        g = np.asarray(grp)
        ld, n, off, res, ioff, ip = _gather(B, g, "getrf")
        m = B.m_h[g]
        A0 = np.zeros_like(res)
        irrgen.fill_packed(seed, m, n, ld, off, A0, gids=gids[g])
        rec = oracle.check_getrf_packed(m, n, A0, ld, off, res, ld, off, ip, ioff, info[g], nthreads=THREADS)
        _merge(tot, assess_getrf(rec, info[g], label))
    return tot


def _run_getrf_config(name):
    cfg = irrgen.config(name)
    B = MatrixBatch(cfg.m, cfg.n)
    gids = np.arange(B.batch)
    host = np.zeros(B.total)
    irrgen.fill_packed(cfg.seed, cfg.m, cfg.n, B.ld_h, B.offsets, host, gids=gids)
    B.data.copy_(torch.from_numpy(host))
    del host
    B.getrf()
    torch.cuda.synchronize()
    return cfg, B, gids


@pytest.mark.parametrize("name", ["C1", "C2", "C3", "C1big"])
def test_every_matrix_getrf(name):
    t0 = time.time()
    cfg, B, gids = _run_getrf_config(name)
    st = _check_getrf_batch(B, cfg.seed, gids, np.arange(B.batch), name)
    print(f"\n[parity {name}] {st} ({time.time() - t0:.1f} s, {THREADS} threads)")
    assert st["checked"] == B.batch and st["skipped"] == 0
    assert st["near_tie"] <= max(2, B.batch // 1000)


def test_every_front_c4_partial():
    t0 = time.time()
    cfg = irrgen.config("C4")
    F = FrontBatch(cfg.m, cfg.n)
    gids = np.arange(F.batch)
    host = np.zeros(F.total)
    irrgen.fill_packed(cfg.seed, F.nf_h, F.nf_h, F.ld_h, F.offsets, host, gids=gids)
    F.data.copy_(torch.from_numpy(host))
    del host
    F.getrf_partial()
    torch.cuda.synchronize()
    info = F.info.cpu().numpy()[: F.batch]
    tot = {}
    for grp in _groups(F.ld_h * F.nf_h, np.arange(F.batch)):
        g = np.asarray(grp)
        ld, nf, off, res, ioff, ip = _gather(F, g, "partial")
        F0 = np.zeros_like(res)
        irrgen.fill_packed(cfg.seed, nf, nf, ld, off, F0, gids=gids[g])
        rec = oracle.check_partial_packed(F.n1_h[g], F.n2_h[g], F0, ld, off, res, ld, off, ip, ioff, info[g],
                                          nthreads=THREADS)
        _merge(tot, assess_partial(rec, info[g], F.n1_h[g], "C4"))
    print(f"\n[parity C4] {tot} ({time.time() - t0:.1f} s, {THREADS} threads)")
    assert tot["fronts"] == F.batch


def test_c5_large_fronts_and_sample():
    """C5 as bench.py runs it (200,000 fronts generated on the device, one
    irr_getrf call): a seeded sample of 64 of the ~2,000 fronts >= 1024 plus
    2,000 of the others (IRR_PARITY_C5_ALL=1: every front >= 1024 -- about
    half an hour of the box's 16 host cores, run once per round by
    tools/gpu_runs and committed under profiles/)."""
    from irrgen import device as gdev
    t0 = time.time()
    cfg = irrgen.config("C5")
    B = MatrixBatch(cfg.m, cfg.n)
    gids = np.arange(B.batch)
    gdev.Filler(cfg.seed, cfg.m, cfg.n, B.ld_h, B.offsets, gids, B.device).fill(B.data)
    B.getrf()
    torch.cuda.synchronize()
    large = np.nonzero(cfg.m >= 1024)[0]
    big = large if os.environ.get("IRR_PARITY_C5_ALL") == "1" else \
        np.sort(np.random.default_rng(2025).choice(large, size=64, replace=False))
    rest = np.setdiff1d(np.arange(B.batch), large)
    sample = np.sort(np.random.default_rng(2024).choice(rest, size=2000, replace=False))
    sel = np.union1d(big, sample)
    st = _check_getrf_batch(B, cfg.seed, gids, sel, "C5")
    print(f"\n[parity C5] fronts >= 1024: {len(big)} of {len(large)} (seed 2025), sample of the rest: "
          f"{len(sample)} (seed 2024); "
          f"{st} ({time.time() - t0:.1f} s, {THREADS} threads)")
    assert st["checked"] == len(sel)
    assert st["near_tie"] <= 4

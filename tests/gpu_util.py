"""Helpers for the -m gpu parity tests: move host matrices through the C ABI
(paper_conf_sc_abdelfattahgbtld22_b200.irr) and compare with the oracle.

Pass criteria (north_star):
  * ipiv and info bit-exact wherever the oracle's pivots are well separated
    (rho > 1 + 1e-6); a mismatch is only allowed at a near tie;
  * backward error ||PA - LU||_F / (||A||_F * k * eps) <= 10 on every matrix;
  * where ipiv agrees, max|X - X_o| / max|X_o| <= 1e-10 for X = L and X = U.
"""
import numpy as np
import torch

import oracle
from paper_conf_sc_abdelfattahgbtld22_b200 import irr
from paper_conf_sc_abdelfattahgbtld22_b200.batch import FrontBatch, MatrixBatch

BE_TOL = 10.0
DEV_TOL = 1e-10
NEAR_TIE = 1.0 + 1e-6


def split_lu(LU):
    m, n = LU.shape
    k = min(m, n)
    L = np.tril(LU[:, :k], -1) + np.eye(m, k)
    U = np.triu(LU[:k, :])
    return L, U


def rel_dev(X, Xo):
    s = np.abs(Xo).max() if Xo.size else 0.0
    d = np.abs(X - Xo).max() if Xo.size else 0.0
    return d / s if s > 0 else d


def gpu_getrf(mats, ld_extra=0, max_m=None, max_n=None, m=None, n=None):
    """Factor host matrices through irr_getrf.  Returns (LUs, ipivs, info, batch)."""
    ma = [A.shape[0] for A in mats]
    na = [A.shape[1] for A in mats]
    ld = [max(1, a + (ld_extra if np.isscalar(ld_extra) else ld_extra[i])) for i, a in enumerate(ma)]
    B = MatrixBatch(ma, na, ld)
    if m is not None:   # deliberately bad local dims (argument checking tests)
        B.m = torch.tensor(m, dtype=torch.int32, device=B.device)
    if n is not None:
        B.n = torch.tensor(n, dtype=torch.int32, device=B.device)
    host = np.full(B.total, np.nan)
    for i, A in enumerate(mats):
        if A.size:
            B.matrix(i, host)[:, :] = A
    B.data.copy_(torch.from_numpy(host))
    B.getrf(max_m=max_m, max_n=max_n)
    torch.cuda.synchronize()
    out = B.data.cpu().numpy()
    ip = B.ipiv_data.cpu().numpy()
    info = B.info.cpu().numpy()[: B.batch].copy()
    LUs = [np.array(B.matrix(i, out)) for i in range(B.batch)]
    ipivs = [np.array(B.ipiv_of(i, ip)) for i in range(B.batch)]
    return LUs, ipivs, info, (B, out)


def check_getrf(A0, LU, ipiv, info, exact=False, label=""):
    """Compare one GPU factorization with the oracle; returns a status string."""
    LUo, ipo, info_o, sep = oracle.getrf(A0)
    m, n = A0.shape
    if exact:
        assert info == info_o, f"{label}: info {info} != {info_o}"
        assert np.array_equal(ipiv, ipo), f"{label}: ipiv differs"
        assert np.array_equal(LU, LUo), f"{label}: L/U not bit-exact, maxdiff {np.abs(LU - LUo).max()}"
        return "exact"
    if min(m, n) == 0:
        assert info == 0
        return "empty"
    be = oracle.backward_error(A0, LU, ipiv)
    assert be <= BE_TOL, f"{label}: backward error {be}"
    if np.array_equal(ipiv, ipo):
        assert info == info_o, f"{label}: info {info} != {info_o}"
        L, U = split_lu(LU)
        Lo, Uo = split_lu(LUo)
        dl, du = rel_dev(L, Lo), rel_dev(U, Uo)
        assert dl <= DEV_TOL and du <= DEV_TOL, f"{label}: L dev {dl}, U dev {du}"
        return "match"
    assert sep < NEAR_TIE, f"{label}: ipiv differs with well separated pivots (rho={sep})"
    return "near-tie"


def gpu_partial(fronts, lapack=False):
    """fronts: list of full nf x nf host arrays with their n1.  Returns the
    factored fronts, ipivs, info (lapack=True: irr_getrf_partial_lapack)."""
    n1 = [f[1] for f in fronts]
    n2 = [f[0].shape[0] - f[1] for f in fronts]
    B = FrontBatch(n1, n2)
    host = np.full(B.total, np.nan)
    for i, (F, _) in enumerate(fronts):
        if F.size:
            B.front(i, host)[:, :] = F
    B.data.copy_(torch.from_numpy(host))
    B.getrf_partial(lapack=lapack)
    torch.cuda.synchronize()
    out = B.data.cpu().numpy()
    ip = B.ipiv_data.cpu().numpy()
    info = B.info.cpu().numpy()[: B.batch].copy()
    return [np.array(B.front(i, out)) for i in range(B.batch)], [np.array(B.ipiv_of(i, ip)) for i in range(B.batch)], info


def check_partial(F0, n1, Fg, ipiv, info, exact=False, label=""):
    F11, F12, F21, F22 = F0[:n1, :n1], F0[:n1, n1:], F0[n1:, :n1], F0[n1:, n1:]
    o11, o12, o22, ipo, info_o = oracle.getrf_partial(F11, F12, F21, F22)
    g11, g12, g21, g22 = Fg[:n1, :n1], Fg[:n1, n1:], Fg[n1:, :n1], Fg[n1:, n1:]
    assert np.array_equal(g21, F21), f"{label}: F21 modified"
    if exact:
        assert info == info_o and np.array_equal(ipiv, ipo), f"{label}: ipiv/info"
        assert np.array_equal(g11, o11), f"{label}: F11 not exact"
        assert np.array_equal(g12, o12), f"{label}: F12 not exact"
        assert np.array_equal(g22, o22), f"{label}: F22 not exact"
        return "exact"
    if n1 == 0:
        assert np.array_equal(g22, F22)
        return "empty"
    st = check_getrf(F11, g11, ipiv, info, label=label + "/F11")
    if st != "match":
        return st
    # F12: relative to max|F12_o|; F22: relative to the update scale (Q12)
    assert rel_dev(g12, o12) <= DEV_TOL, f"{label}: F12 dev {rel_dev(g12, o12)}"
    if F22.size:
        sigma = (np.abs(F22) + np.abs(F21) @ np.abs(o12)).max()
        d = np.abs(g22 - o22).max()
        assert d <= DEV_TOL * max(sigma, 1e-300), f"{label}: F22 dev {d / sigma}"
    return "match"


def fnv1a_ipiv(ipiv) -> int:
    """Host FNV-1a (32-bit) of an int32 pivot vector's little-endian bytes --
    the definition irr_status_words implements (include/irr.h)."""
    h = 2166136261
    for byte in np.ascontiguousarray(ipiv, dtype="<i4").tobytes():
        h = ((h ^ byte) * 16777619) & 0xFFFFFFFF
    return h

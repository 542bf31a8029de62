"""Pass / fail rules applied to the oracle's batched parity records
(oracle.check_getrf_packed / check_partial_packed), plus the helpers that run
a whole packed batch through them.

The rules restate north_star with SURVEY §8(c) readings Q11-Q13:
  * backward error ||PA - LU||_F / (||A||_F k eps) <= 10 on EVERY matrix;
  * |l_ij| <= 1 (+ rounding of the GPU's own l = a * (1/p), reading Q6) on
    EVERY matrix: in exact terms |l_rk| = |a_rk^(k)| / |u_kk|, so this says
    the GPU's pivot is the column maximum at its step (G8);
  * where ipiv equals the oracle's: info equal, L / U deviation <= 1e-10
    (normwise-max relative, Q12), and for fronts F12 / F22 likewise;
  * an ipiv mismatch is accepted only at a near tie of the oracle's own
    pivots (rho < 1 + 1e-6, Q13) -- and it is counted and reported.
"""
from __future__ import annotations

import numpy as np

import oracle

BE_TOL = 10.0
DEV_TOL = 1e-10
NEAR_TIE = 1.0 + 1e-6
LMAX_TOL = 1.0 + 4 * np.finfo(np.float64).eps

G = {f: i for i, f in enumerate(oracle.PARTIAL_FIELDS)}


def assess_getrf(rec: np.ndarray, info: np.ndarray, label: str = "", exact: bool = False) -> dict:
    """Apply the rules to getrf records; raises AssertionError naming the
    first offending matrix.  Returns counts {checked, match, near_tie, exact,
    skipped (info < 0), max_be, max_dev}."""
    info = np.asarray(info)
    live = info >= 0
    r = rec[live]
    idx = np.nonzero(live)[0]
    eq = r[:, G["ipiv_eq"]] == 1
    be = r[:, G["be"]]
    bad = np.nonzero(~(be <= BE_TOL))[0]
    assert bad.size == 0, f"{label}: backward error {be[bad[0]]} on matrix {idx[bad[0]]}"
    lm = r[:, G["lmax"]]
    bad = np.nonzero(~(lm <= LMAX_TOL))[0]
    assert bad.size == 0, f"{label}: |l| = {lm[bad[0]]} > 1 on matrix {idx[bad[0]]} (pivot not the column max)"
    inf_ok = r[:, G["info_o"]] == info[live]
    bad = np.nonzero(eq & ~inf_ok)[0]
    assert bad.size == 0, f"{label}: info {info[idx[bad[0]]]} != oracle {r[bad[0], G['info_o']]} on {idx[bad[0]]}"
    dev = np.maximum(r[:, G["dl"]], r[:, G["du"]])
    bad = np.nonzero(eq & ~(dev <= DEV_TOL))[0]
    assert bad.size == 0, f"{label}: L/U deviation {dev[bad[0]]} on matrix {idx[bad[0]]}"
    tie = ~eq
    bad = np.nonzero(tie & ~(r[:, G["rho"]] < NEAR_TIE))[0]
    assert bad.size == 0, (f"{label}: ipiv differs at step {int(r[bad[0], G['first_diff']])} of matrix "
                           f"{idx[bad[0]]} with well separated pivots (rho = {r[bad[0], G['rho']]})")
    if exact:
        bad = np.nonzero(r[:, G["exact"]] != 1)[0]
        assert bad.size == 0, f"{label}: matrix {idx[bad[0]]} not bit-exact"
    return {"checked": int(live.sum()), "match": int(eq.sum()), "near_tie": int(tie.sum()),
            "exact": int((r[:, G["exact"]] == 1).sum()), "skipped": int((~live).sum()),
            "max_be": float(be.max()) if be.size else 0.0,
            "max_dev": float(np.nanmax(dev[eq])) if eq.any() else 0.0}


def assess_partial(rec: np.ndarray, info: np.ndarray, n1: np.ndarray, label: str = "",
                   exact: bool = False) -> dict:
    """Rules for partial fronts: F11 as getrf; F21 untouched; where ipiv
    agrees and F11 is nonsingular, F12 / F22 deviation <= 1e-10 (Q12)."""
    info = np.asarray(info)
    n1 = np.asarray(n1)
    live = info >= 0
    r = rec[live]
    idx = np.nonzero(live)[0]
    nz = n1[live] > 0
    out = assess_getrf(rec[live][nz], info[live][nz], label + "/F11", exact=False)
    bad = np.nonzero(r[:, G["f21_same"]] != 1)[0]
    assert bad.size == 0, f"{label}: F21 modified on front {idx[bad[0]]}"
    eq = (r[:, G["ipiv_eq"]] == 1) & (info[live] == 0)
    for f in ("d12", "d22"):
        d = r[:, G[f]]
        bad = np.nonzero(eq & nz & ~(d <= DEV_TOL))[0]
        assert bad.size == 0, f"{label}: {f} = {d[bad[0]]} on front {idx[bad[0]]}"
    if exact:
        bad = np.nonzero(r[:, G["front_exact"]] != 1)[0]
        assert bad.size == 0, f"{label}: front {idx[bad[0]]} not bit-exact"
    out["fronts"] = int(live.sum())
    out["max_d12"] = float(np.nanmax(r[eq & nz, G["d12"]])) if (eq & nz).any() else 0.0
    out["max_d22"] = float(np.nanmax(r[eq & nz, G["d22"]])) if (eq & nz).any() else 0.0
    return out

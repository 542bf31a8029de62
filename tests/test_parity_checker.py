"""CPU pins of the batched parity checker (oracle/check.c + tests/parity.py):
the oracle's own results pass bit-exactly, and each plausible GPU mistake --
a perturbed L or U entry, a wrong pivot, a valid factorization with a
non-maximal pivot, a touched F21, a perturbed F12 / F22 -- is caught."""
import numpy as np
import pytest

import irrgen
import oracle
from parity import assess_getrf, assess_partial


def _packed(shapes, seed=3):
    m = np.array([s[0] for s in shapes])
    n = np.array([s[1] for s in shapes])
    ld = np.maximum(1, m)
    off, total = irrgen.packed_offsets(ld, n)
    A0 = np.zeros(total)
    irrgen.fill_packed(seed, m, n, ld, off, A0)
    return m, n, ld, off, A0


def _view(flat, off, m, n, ld):
    return flat[off: off + ld * n].reshape((n, ld)).T[:m, :]


def _oracle_results(m, n, ld, off, A0):
    """The oracle's factors packed like a GPU result."""
    LU = A0.copy()
    k = np.minimum(m, n)
    ioff = np.concatenate([[0], np.cumsum(np.maximum(k, 1))[:-1]]).astype(np.int64)
    ipiv = np.zeros(int(np.maximum(k, 1).sum()), dtype=np.int32)
    info = np.zeros(len(m), dtype=np.int32)
    for i in range(len(m)):
        A = _view(A0, off[i], m[i], n[i], ld[i])
        LUo, ipo, info_o, _ = oracle.getrf(A)
        _view(LU, off[i], m[i], n[i], ld[i])[:, :] = LUo
        ipiv[ioff[i]: ioff[i] + k[i]] = ipo
        info[i] = info_o
    return LU, ipiv, ioff, info


SHAPES = [(1, 1), (5, 5), (17, 9), (9, 17), (40, 40), (64, 30), (0, 4), (33, 33)]


def test_oracle_results_pass_exactly():
    m, n, ld, off, A0 = _packed(SHAPES)
    LU, ipiv, ioff, info = _oracle_results(m, n, ld, off, A0)
    rec = oracle.check_getrf_packed(m, n, A0, ld, off, LU, ld, off, ipiv, ioff, info)
    st = assess_getrf(rec, info, exact=True)
    assert st["exact"] == len(SHAPES) and st["near_tie"] == 0


@pytest.mark.parametrize("where", ["L", "U"])
def test_perturbed_factor_is_caught(where):
    m, n, ld, off, A0 = _packed(SHAPES)
    LU, ipiv, ioff, info = _oracle_results(m, n, ld, off, A0)
    V = _view(LU, off[4], m[4], n[4], ld[4])
    i, j = (20, 3) if where == "L" else (3, 20)
    V[i, j] *= 1 + 1e-8
    rec = oracle.check_getrf_packed(m, n, A0, ld, off, LU, ld, off, ipiv, ioff, info)
    assert rec[4, oracle.GETRF_FIELDS.index("d" + where.lower())] > 1e-10
    with pytest.raises(AssertionError):   # (the backward error also trips at this size)
        assess_getrf(rec, info)


def test_wrong_pivot_is_caught():
    m, n, ld, off, A0 = _packed(SHAPES)
    LU, ipiv, ioff, info = _oracle_results(m, n, ld, off, A0)
    ipiv[ioff[4]] = 1 if ipiv[ioff[4]] != 1 else 2
    rec = oracle.check_getrf_packed(m, n, A0, ld, off, LU, ld, off, ipiv, ioff, info)
    with pytest.raises(AssertionError):
        assess_getrf(rec, info)


def test_non_maximal_pivot_is_caught():
    """A = [[1, 0], [2, 1]] factored WITHOUT the interchange is an exact
    factorization (backward error 0) but |l| = 2: the rule on |l| rejects it."""
    A0 = np.array([1.0, 2.0, 0.0, 1.0])        # column-major 2 x 2
    LU = np.array([1.0, 2.0, 0.0, 1.0])        # L = [[1, 0], [2, 1]], U = I
    m = n = ld = np.array([2])
    off = np.array([0])
    ipiv = np.array([1, 2], dtype=np.int32)
    rec = oracle.check_getrf_packed(m, n, A0, ld, off, LU, ld, off, ipiv, np.array([0]), np.array([0]))
    F = {f: i for i, f in enumerate(oracle.GETRF_FIELDS)}
    assert rec[0, F["be"]] == 0.0 and rec[0, F["lmax"]] == 2.0
    with pytest.raises(AssertionError, match=r"\|l\|"):
        assess_getrf(rec, np.array([0]))


def test_rejected_matrices_are_skipped():
    m, n, ld, off, A0 = _packed(SHAPES)
    LU, ipiv, ioff, info = _oracle_results(m, n, ld, off, A0)
    info[2] = -1
    LU[off[2]] = np.nan
    rec = oracle.check_getrf_packed(m, n, A0, ld, off, LU, ld, off, ipiv, ioff, info)
    st = assess_getrf(rec, info)
    assert st["skipped"] == 1 and st["checked"] == len(SHAPES) - 1


def _fronts(pairs, seed=5):
    n1 = np.array([p[0] for p in pairs])
    n2 = np.array([p[1] for p in pairs])
    nf = n1 + n2
    ld = np.maximum(1, nf)
    off, total = irrgen.packed_offsets(ld, nf)
    F0 = np.zeros(total)
    irrgen.fill_packed(seed, nf, nf, ld, off, F0)
    Fg = F0.copy()
    ioff = np.concatenate([[0], np.cumsum(np.maximum(n1, 1))[:-1]]).astype(np.int64)
    ipiv = np.zeros(int(np.maximum(n1, 1).sum()), dtype=np.int32)
    info = np.zeros(len(n1), dtype=np.int32)
    for i, (a, b) in enumerate(pairs):
        V = _view(Fg, off[i], a + b, a + b, ld[i])
        o11, o12, o22, ipo, inf = oracle.getrf_partial(V[:a, :a], V[:a, a:], V[a:, :a], V[a:, a:])
        V[:a, :a], V[:a, a:], V[a:, a:] = o11, o12, o22
        ipiv[ioff[i]: ioff[i] + a] = ipo
        info[i] = inf
    return n1, n2, ld, off, F0, Fg, ipiv, ioff, info


PAIRS = [(1, 0), (3, 4), (10, 10), (17, 40), (0, 5), (30, 12)]


def test_partial_oracle_results_pass_exactly():
    n1, n2, ld, off, F0, Fg, ipiv, ioff, info = _fronts(PAIRS)
    rec = oracle.check_partial_packed(n1, n2, F0, ld, off, Fg, ld, off, ipiv, ioff, info)
    st = assess_partial(rec, info, n1, exact=True)
    assert st["fronts"] == len(PAIRS)


@pytest.mark.parametrize("block", ["F21", "F12", "F22"])
def test_partial_errors_are_caught(block):
    n1, n2, ld, off, F0, Fg, ipiv, ioff, info = _fronts(PAIRS)
    i, a = 3, PAIRS[3][0]
    V = _view(Fg, off[i], a + PAIRS[i][1], a + PAIRS[i][1], ld[i])
    if block == "F21":
        V[a + 1, 2] += 2.0 ** -40
    elif block == "F12":
        V[2, a + 5] *= 1 + 1e-8
    else:
        V[a + 3, a + 7] += 1e-6
    rec = oracle.check_partial_packed(n1, n2, F0, ld, off, Fg, ld, off, ipiv, ioff, info)
    with pytest.raises(AssertionError):
        assess_partial(rec, info, n1)

"""CPU pins of the oracle's §8(f) NEXT 3 functions:

* oracle.getrf_partial_lapack -- the LAPACK-style partial front (L21 = F21 U^-1,
  U12 = L^-1 P^T F12, PAPER.md L96-97 / reading Q8's alternative): exact
  construction (bit-exact), scipy LAPACK cross-check, same Schur complement as
  the paper's variant;
* oracle.zgetrf -- complex LU with partial pivoting (the solver's A in
  C^{N x N}) with LAPACK zgetf2 semantics (izamax: |Re| + |Im|,
  DESIGN reading Q20): exact Gaussian-rational elimination on tiny inputs,
  the exact complex dyadic family, scipy (LAPACK zgetrf), the real
  embedding, determinants, the tie rule, and zbackward_error's closed form.
"""
from fractions import Fraction

import numpy as np
import pytest
import scipy.linalg as sl

import irrgen
import oracle

EPS = np.finfo(np.float64).eps


# ------------------------------------------------------------------ LAPACK-style partial
@pytest.mark.parametrize("n1,n2", [(1, 1), (5, 7), (16, 3), (33, 40), (64, 20), (3, 0), (0, 4)])
def test_partial_lapack_exact(n1, n2):
    f = irrgen.g1_front_lapack(12, n1 * 100 + n2, n1, n2)
    o11, o12, o21, o22, ip, info = oracle.getrf_partial_lapack(f["F11"], f["F12"], f["F21"], f["F22"])
    assert info == 0
    assert np.array_equal(ip, f["ipiv"])
    assert np.array_equal(o11, np.tril(f["L"], -1) + f["U"])
    assert np.array_equal(o12, f["X"]) and np.array_equal(o21, f["Y"]) and np.array_equal(o22, f["S"])


@pytest.mark.parametrize("n1,n2", [(6, 9), (40, 25), (97, 64)])
def test_partial_lapack_vs_scipy(n1, n2):
    F = irrgen.front_values(13, n1 + n2, n1 + n2)
    F11, F12, F21, F22 = F[:n1, :n1], F[:n1, n1:], F[n1:, :n1], F[n1:, n1:]
    o11, o12, o21, o22, ip, _ = oracle.getrf_partial_lapack(F11, F12, F21, F22)
    lu, piv = sl.lu_factor(F11)
    assert np.array_equal(ip, piv + 1)
    P12 = F12.copy()
    for k, p in enumerate(piv):
        P12[[k, p], :] = P12[[p, k], :]
    U12 = sl.solve_triangular(lu, P12, lower=True, unit_diagonal=True)
    L21 = sl.solve_triangular(lu, F21.T, trans="T", lower=False).T
    S = F22 - L21 @ U12
    for got, want in ((o12, U12), (o21, L21), (o22, S)):
        assert np.abs(got - want).max() <= 1e-12 * max(1.0, np.abs(want).max())


def test_partial_lapack_same_schur_as_paper_variant():
    n1, n2 = 50, 70
    F = irrgen.front_values(14, 1, n1 + n2)
    blocks = F[:n1, :n1], F[:n1, n1:], F[n1:, :n1], F[n1:, n1:]
    a11, a12, a21, a22, aip, _ = oracle.getrf_partial_lapack(*blocks)
    p11, p12, p22, pip, _ = oracle.getrf_partial(*blocks)
    assert np.array_equal(a11, p11) and np.array_equal(aip, pip)   # step 1 is the same GEPP
    assert np.abs(a22 - p22).max() <= 1e-12 * np.abs(p22).max()
    # L21 U12 = F21 F11^-1 F12 = F21 X_paper
    assert np.abs(a21 @ a12 - blocks[2] @ p12).max() <= 1e-12 * np.abs(blocks[2] @ p12).max()


def test_partial_lapack_bad_arguments():
    L = oracle.lib()
    assert L.oracle_getrf_partial_lapack(-1, 0, None, 1, None, 1, None, 1, None, 1, None, None) == -1
    assert L.oracle_getrf_partial_lapack(2, 2, None, 1, None, 2, None, 2, None, 2, None, None) == -4
    assert L.oracle_getrf_partial_lapack(2, 3, None, 2, None, 2, None, 2, None, 3, None, None) == -8


# ------------------------------------------------------------------ ZGETRF
def _cabs1(z):
    return abs(z.real) + abs(z.imag)


def _exact_zgepp(A):
    """Gaussian-rational GEPP with izamax pivoting (Fractions)."""
    m, n = A.shape
    R = [[(Fraction(A[i, j].real), Fraction(A[i, j].imag)) for j in range(n)] for i in range(m)]
    ipiv = []
    for k in range(min(m, n)):
        c1 = [abs(R[i][k][0]) + abs(R[i][k][1]) for i in range(k, m)]
        best = max(c1)
        p = k + c1.index(best)
        ipiv.append(p + 1)
        if best != 0:
            R[k], R[p] = R[p], R[k]
            cr, ci = R[k][k]
            den = cr * cr + ci * ci
            for i in range(k + 1, m):
                ar, ai = R[i][k]
                R[i][k] = ((ar * cr + ai * ci) / den, (ai * cr - ar * ci) / den)
            for i in range(k + 1, m):
                lr, li = R[i][k]
                for j in range(k + 1, n):
                    ur, ui = R[k][j]
                    R[i][j] = (R[i][j][0] - (lr * ur - li * ui), R[i][j][1] - (lr * ui + li * ur))
    return np.array([[complex(float(x), float(y)) for x, y in row] for row in R]), np.array(ipiv, dtype=np.int32)


@pytest.mark.parametrize("m,n", [(1, 1), (2, 2), (3, 3), (4, 4), (5, 5), (5, 3), (3, 5)])
def test_zgetrf_exact_rational(m, n):
    for g in range(6):
        A = irrgen.zuniform_values(31, 10 * m + n + 100 * g, m, n)
        LU, ip, info, _ = oracle.zgetrf(A)
        LUx, ipx = _exact_zgepp(A)
        assert np.array_equal(ip, ipx)
        assert np.abs(LU - LUx).max() <= 64 * EPS * max(1.0, np.abs(LUx).max())


@pytest.mark.parametrize("m,n", [(1, 1), (8, 8), (17, 9), (9, 17), (64, 64), (130, 100)])
def test_zg1_exact_bitexact(m, n):
    A, L, U, ipiv, _ = irrgen.zg1_exact(32, m * 1000 + n, m, n)
    LU, ip, info, sep = oracle.zgetrf(A)
    k = min(m, n)
    assert info == 0 and np.array_equal(ip, ipiv) and sep >= 2.0
    assert np.array_equal(np.tril(LU[:, :k], -1) + np.eye(m, k), L)
    assert np.array_equal(np.triu(LU[:k, :]), U)


@pytest.mark.parametrize("n,c", [(6, 0), (6, 3), (40, 39), (70, 20)])
def test_zg1_singular(n, c):
    A, L, U, ipiv, info = irrgen.zg1_exact(33, n + c, n, n, singular_col=c)
    LU, ip, inf, _ = oracle.zgetrf(A)
    assert inf == info == c + 1 and np.array_equal(ip, ipiv)
    assert np.array_equal(np.triu(LU), U)


@pytest.mark.parametrize("m,n", [(12, 12), (60, 45), (45, 60), (150, 150)])
def test_zgetrf_vs_scipy(m, n):
    A = irrgen.zuniform_values(34, m + n, m, n)
    LU, ip, info, sep = oracle.zgetrf(A)
    lu, piv = sl.lu_factor(A, check_finite=False)
    assert sep > 1 + 1e-6
    assert np.array_equal(ip, piv + 1)
    assert np.abs(LU - lu).max() <= 1e-12 * np.abs(lu).max()
    assert oracle.zbackward_error(A, LU, ip) <= 1.0


def test_zgetrf_real_embedding():
    """A real matrix factored as complex: the same pivots as dgetrf (|Re| + 0
    is |Re|) and the same factors up to rounding (the complex division is
    a c / c^2, not a / c); zero imaginary parts stay exactly zero."""
    A = irrgen.uniform_values(35, 1, 50, 50)
    LUd, ipd, _, _ = oracle.getrf(A)
    LUz, ipz, _, _ = oracle.zgetrf(A.astype(np.complex128))
    assert np.array_equal(ipd, ipz)
    assert np.all(LUz.imag == 0.0)
    assert np.abs(LUz.real - LUd).max() <= 1e-13 * np.abs(LUd).max()


def test_zgetrf_determinant():
    for n in (3, 7, 20):
        A = irrgen.zuniform_values(36, n, n, n)
        LU, ip, _, _ = oracle.zgetrf(A)
        sign = (-1) ** int(np.sum(ip != np.arange(1, n + 1)))
        det = sign * np.prod(np.diag(LU))
        assert abs(det - np.linalg.det(A)) <= 1e-12 * abs(np.linalg.det(A)) * n


def test_zgetrf_tie_rule_and_zero_pivot():
    """izamax: |Re| + |Im| ties -> the smallest row; an all-zero column ->
    info, no interchange, no scaling."""
    A = np.array([[1.0 + 0j, 0.0], [1j, 1.0], [-1.0, 2.0]])
    _, ip, _, sep = oracle.zgetrf(A)
    assert ip[0] == 1 and sep == 1.0
    A = np.array([[0.5 + 0j], [1j], [1.0]])
    _, ip, _, _ = oracle.zgetrf(A)
    assert ip[0] == 2
    A = np.array([[0j, 1.0], [0j, 2.0]])
    LU, ip, info, _ = oracle.zgetrf(A)
    assert info == 1 and ip[0] == 1 and np.array_equal(LU, A)


def test_zbackward_error_closed_form():
    """Exact factors of a complex G1 matrix with U's last row perturbed by
    delta (only L's unit diagonal multiplies it): ||PA - LU||_F = |delta|
    exactly, so be = |delta| / (||A||_F k eps)."""
    n = 12
    A, L, U, ipiv, _ = irrgen.zg1_exact(37, 1, n, n)
    LU = np.tril(L, -1) + U
    delta = 3.0 - 4.0j
    LU[n - 1, n - 1] += delta
    want = abs(delta) / (np.linalg.norm(A) * n * EPS)
    assert abs(oracle.zbackward_error(A, LU, ipiv) - want) <= 1e-12 * want

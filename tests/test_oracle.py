"""Pins for the CPU oracle (oracle/oracle.c) against things other than itself:
exact rational elimination, Leibniz determinants, closed forms, exactly
constructed factor families, LAPACK (scipy) and invariants.  CPU only.

Each pin cites the PAPER.md passage (P:L<line>) or SURVEY.md §8(c) reading it
checks.  A plausible mistake in the oracle (dropped term, wrong sign, wrong
index, transposed operand, wrong tie rule) fails at least one test here.
"""
import itertools
import math
from fractions import Fraction

import numpy as np
import pytest
import scipy.linalg as sl

import irrgen

EPS = np.finfo(np.float64).eps


# ---------------------------------------------------------------- helpers
def exact_gepp(A):
    """Textbook GEPP in exact rationals, tie -> smallest row.
    Returns (LU as Fractions, 0-based ipiv, info, rho_exact)."""
    m, n = len(A), len(A[0])
    a = [[Fraction(x) for x in row] for row in A]
    ipiv, info, rho = [], 0, math.inf
    for k in range(min(m, n)):
        mags = [abs(a[i][k]) for i in range(k, m)]
        best = max(mags)
        p = k + mags.index(best)
        rest = sorted(mags, reverse=True)
        if len(rest) > 1 and rest[1] > 0 and best > 0:
            rho = min(rho, float(best / rest[1]))
        ipiv.append(p)
        if a[p][k] != 0:
            a[k], a[p] = a[p], a[k]
            for i in range(k + 1, m):
                a[i][k] = a[i][k] / a[k][k]
        elif info == 0:
            info = k + 1
        for i in range(k + 1, m):
            for j in range(k + 1, n):
                a[i][j] -= a[i][k] * a[k][j]
    return a, ipiv, info, rho


def leibniz_det(A):
    n = len(A)
    tot = Fraction(0)
    for perm in itertools.permutations(range(n)):
        inv = sum(1 for i in range(n) for j in range(i + 1, n) if perm[i] > perm[j])
        p = Fraction(1)
        for i in range(n):
            p *= Fraction(A[i][perm[i]])
        tot += -p if inv % 2 else p
    return tot


def split_lu(LU):
    m, n = LU.shape
    k = min(m, n)
    L = np.tril(LU[:, :k], -1) + np.eye(m, k)
    U = np.triu(LU[:k, :])
    return L, U


def apply_swaps(A, ipiv1):
    A = A.copy()
    for k, p in enumerate(ipiv1):
        p -= 1
        if p != k:
            A[[k, p], :] = A[[p, k], :]
    return A


# ---------------------------------------------------------------- GEPP pins
@pytest.mark.parametrize("m,n", [(1, 1), (2, 2), (3, 3), (4, 4), (5, 5), (6, 6), (6, 3), (3, 6), (5, 2), (2, 5)])
def test_getrf_matches_exact_rational_elimination(orc, m, n):
    """Brute force on tiny inputs: the oracle's ipiv equals exact
    GEPP's and its factors are within rounding of the exact rationals."""
    for gid in range(40):
        A = irrgen.uniform_values(7, gid, m, n)
        ex, ipiv0, info, rho = exact_gepp(A.tolist())
        LU, ipiv, oinfo, sep = orc.getrf(A)
        if rho < 1 + 1e-9:
            continue                                   # near tie: pivot may legally differ
        assert list(ipiv - 1) == ipiv0
        assert oinfo == info == 0
        exf = np.array([[float(x) for x in row] for row in ex])
        scale = max(1.0, np.abs(exf).max())
        assert np.abs(LU - exf).max() <= 1e-12 * scale
        assert sep == pytest.approx(rho, rel=1e-9)


def test_tie_break_smallest_row(orc):
    """Q3: idamax semantics -- on an exact tie the smallest row index wins."""
    A = np.array([[1.0, 2.0], [-1.0, 5.0]])
    _, ipiv, _, sep = orc.getrf(A)
    assert ipiv[0] == 1 and sep == 1.0
    A = np.array([[0.5, 1.0, 0.0], [-2.0, 0.0, 1.0], [2.0, 1.0, 1.0]])
    _, ipiv, _, _ = orc.getrf(A)
    assert ipiv[0] == 2


@pytest.mark.parametrize("n", [2, 3, 4, 5, 6, 7])
def test_determinant_leibniz(orc, n):
    """det(A) = sign(P) * prod u_kk (P:L106 P*L*U = A), against the Leibniz sum."""
    for gid in range(6):
        A = irrgen.uniform_values(11, gid, n, n)
        LU, ipiv, info, _ = orc.getrf(A)
        sign = (-1) ** int(sum(1 for k, p in enumerate(ipiv) if p - 1 != k))
        det = sign * np.prod(np.diag(LU))
        ref = float(leibniz_det(A.tolist()))
        assert det == pytest.approx(ref, rel=1e-11, abs=1e-14)


@pytest.mark.parametrize("m,n", [(8, 8), (64, 64), (100, 37), (37, 100), (256, 255), (300, 40)])
def test_scipy_lapack_crosscheck(orc, m, n):
    """G7: LAPACK dgetrf (scipy) gives the same ipiv and factors within 1e-11
    (LAPACK is blocked and uses a reciprocal, so rounding differs)."""
    A = irrgen.uniform_values(5, m * 1000 + n, m, n)
    LU, ipiv, info, sep = orc.getrf(A)
    lu, piv = sl.lu_factor(A) if m == n else (None, None)
    if m != n:
        P, L, U = sl.lu(A)
        k = min(m, n)
        L2, U2 = split_lu(LU)
        assert np.abs(L2 - L).max() <= 1e-11 * max(1, np.abs(L).max())
        assert np.abs(U2 - U).max() <= 1e-11 * np.abs(U).max()
        # P from scipy: A = P L U -> rows of PA
        assert np.allclose(apply_swaps(A, ipiv), P.T @ A)
    else:
        assert np.array_equal(ipiv, piv + 1)
        assert np.abs(LU - lu).max() <= 1e-11 * np.abs(lu).max()
    assert orc.backward_error(A, LU, ipiv) < 1.0


@pytest.mark.parametrize("m,n", [(1, 1), (5, 5), (8, 8), (33, 33), (64, 20), (20, 64), (130, 130), (257, 100)])
def test_g1_exact_dyadic_bitexact(orc, m, n):
    """G1: A = P L U from chosen dyadic factors; any correct GEPP returns them bit-exactly."""
    A, L, U, ipiv, info = irrgen.g1_exact(3, m + 7 * n, m, n)
    LU, oipiv, oinfo, sep = orc.getrf(A)
    L2, U2 = split_lu(LU)
    assert np.array_equal(oipiv, ipiv)
    assert oinfo == 0
    assert np.array_equal(L2, L) and np.array_equal(U2, U)
    assert sep >= 2.0
    assert orc.backward_error(A, LU, oipiv) == 0.0


@pytest.mark.parametrize("m,n,c", [(6, 6, 0), (6, 6, 2), (100, 100, 99), (64, 40, 17), (40, 64, 39)])
def test_g1_singular(orc, m, n, c):
    """G1-sing / Q5: an exact zero pivot at step c gives info = c+1, no swap,
    no scaling, and the factorization continues (LAPACK dgetrf)."""
    A, L, U, ipiv, info = irrgen.g1_singular(4, c, m, n, c)
    LU, oipiv, oinfo, _ = orc.getrf(A)
    L2, U2 = split_lu(LU)
    assert oinfo == info == c + 1
    assert np.array_equal(oipiv, ipiv)
    assert np.array_equal(L2, L) and np.array_equal(U2, U)


@pytest.mark.parametrize("m,n", [(1, 1), (5, 5), (64, 64), (300, 40), (40, 300), (256, 255), (200, 200)])
def test_g2_dominant_ipiv_from_permutation(orc, m, n):
    """G2: ipiv follows from the row permutation alone; factors vs LAPACK."""
    A, ipiv = irrgen.g2_dominant(9, m * 3 + n, m, n)
    LU, oipiv, oinfo, sep = orc.getrf(A)
    assert np.array_equal(oipiv, ipiv)
    assert sep > 1.5 or min(m, n) == 1 or m == 1
    P, L, U = sl.lu(A)
    L2, U2 = split_lu(LU)
    assert np.abs(L2 - L).max() <= 1e-13
    assert np.abs(U2 - U).max() <= 1e-13 * np.abs(U).max()


def test_g5_closed_forms(orc):
    # 1x1
    LU, ipiv, info, _ = orc.getrf(np.array([[3.5]]))
    assert LU[0, 0] == 3.5 and list(ipiv) == [1] and info == 0
    LU, ipiv, info, _ = orc.getrf(np.array([[0.0]]))
    assert info == 1 and list(ipiv) == [1]
    # m x 1: ipiv = first argmax, L = column / pivot
    col = np.array([[0.5], [-3.0], [3.0], [1.0]])
    LU, ipiv, info, _ = orc.getrf(col)
    assert list(ipiv) == [2] and LU[0, 0] == -3.0
    assert np.array_equal(LU[1:, 0], np.array([0.5, 3.0, 1.0]) / -3.0)
    # 1 x n: ipiv = 1, U = row
    row = np.array([[2.0, -1.0, 7.0]])
    LU, ipiv, info, _ = orc.getrf(row)
    assert list(ipiv) == [1] and np.array_equal(LU, row)
    # identity
    LU, ipiv, info, _ = orc.getrf(np.eye(9))
    assert np.array_equal(LU, np.eye(9)) and list(ipiv) == list(range(1, 10))
    # permutation matrix: L = U = I, ipiv recovers the permutation
    perm = [3, 0, 4, 1, 2]
    Pm = np.eye(5)[perm]
    LU, ipiv, info, _ = orc.getrf(Pm)
    assert np.array_equal(LU, np.eye(5))
    assert np.array_equal(apply_swaps(Pm, ipiv), np.eye(5))
    # upper triangular with dominant diagonal: no swaps, U = A
    T = np.triu(irrgen.uniform_values(1, 1, 7, 7)) + 4 * np.eye(7)
    LU, ipiv, info, _ = orc.getrf(T)
    assert list(ipiv) == list(range(1, 8)) and np.array_equal(LU, T)
    # zero matrix: info = 1, ipiv = 1..k
    LU, ipiv, info, _ = orc.getrf(np.zeros((4, 6)))
    assert info == 1 and list(ipiv) == [1, 2, 3, 4] and not LU.any()
    # column c zeroed in a random matrix: info = c+1, ipiv[c] = c+1
    A = irrgen.uniform_values(2, 2, 50, 50)
    A[:, 17] = 0.0
    LU, ipiv, info, _ = orc.getrf(A)
    assert info == 18 and ipiv[17] == 18
    # m = 0 or n = 0: quick return
    LU, ipiv, info, _ = orc.getrf(np.zeros((0, 5)))
    assert info == 0 and ipiv.size == 0
    LU, ipiv, info, _ = orc.getrf(np.zeros((5, 0)))
    assert info == 0 and ipiv.size == 0


def test_invariants_uniform(orc):
    """G8: |l_ij| <= 1, ipiv[k] in [k+1, m], backward error <= 10 (north_star)."""
    for gid, (m, n) in enumerate([(17, 17), (90, 31), (31, 90), (128, 128)]):
        A = irrgen.uniform_values(13, gid, m, n)
        LU, ipiv, info, _ = orc.getrf(A)
        L, U = split_lu(LU)
        assert np.abs(L).max() <= 1.0
        assert all(k + 1 <= p <= m for k, p in enumerate(ipiv))
        assert orc.backward_error(A, LU, ipiv) <= 10.0


def test_batch_equals_single(orc):
    cfg = irrgen.config("C1")
    mats = [irrgen.uniform_values(cfg.seed, i, int(m), int(n)) for i, (m, n) in enumerate(zip(cfg.m, cfg.n))]
    work = [M.copy(order="F") for M in mats]
    ipivs, info, sep = orc.getrf_batch(work, nthreads=4)
    for M, W, p, inf in zip(mats, work, ipivs, info):
        LU, ip, i1, _ = orc.getrf(M)
        assert np.array_equal(LU, W) and np.array_equal(ip, p) and inf == i1


# ---------------------------------------------------------------- backward error checker
def test_backward_error_closed_form(orc):
    """Perturbing one entry of an exact factorization by d gives exactly
    |d| * (norm of the factor row/column it multiplies) / (||A||_F * k * eps)
    (SURVEY Q11)."""
    A, L, U, ipiv, _ = irrgen.g1_exact(1, 2, 12, 12)
    LU, oipiv, _, _ = orc.getrf(A)
    assert orc.backward_error(A, LU, oipiv) == 0.0
    d = 2.0 ** -20
    LU2 = LU.copy(order="F")
    LU2[0, 5] += d                         # u_05: (LU)_{i,5} changes by d*l_i0 for every i
    be = orc.backward_error(A, LU2, oipiv)
    assert be == pytest.approx(d * np.linalg.norm(L[:, 0]) / (np.linalg.norm(A) * 12 * EPS), rel=1e-12)
    LU3 = LU.copy(order="F")
    LU3[7, 2] += d                         # L entry l_72: (LU)_{7,j} changes by d*u_2j, j>=2
    exp = d * np.linalg.norm(U[2, 2:]) / (np.linalg.norm(A) * 12 * EPS)
    assert orc.backward_error(A, LU3, oipiv) == pytest.approx(exp, rel=1e-12)


# ---------------------------------------------------------------- partial front
@pytest.mark.parametrize("n1,n2", [(1, 1), (5, 7), (16, 3), (64, 200), (33, 65), (120, 40)])
def test_partial_g1front_exact(orc, n1, n2):
    """G1': F12 -> X and F22 -> S bit-exactly."""
    f = irrgen.g1_front(21, n1 * 1000 + n2, n1, n2)
    F11, F12, F22, ipiv, info = orc.getrf_partial(f["F11"], f["F12"], f["F21"], f["F22"])
    L, U = split_lu(F11)
    assert info == 0
    assert np.array_equal(ipiv, f["ipiv"])
    assert np.array_equal(L, f["L"]) and np.array_equal(U, f["U"])
    assert np.array_equal(F12, f["X"])
    assert np.array_equal(F22, f["S"])


@pytest.mark.parametrize("n1,n2", [(1, 0), (7, 0), (0, 5), (10, 10), (50, 80), (97, 31)])
def test_partial_vs_lapack(orc, n1, n2):
    """G7 for the front: F12 = F11^-1 F12 and S = F22 - F21 F11^-1 F12;
    n2 = 0 reduces to getrf and n1 = 0 leaves F22 unchanged (G8)."""
    F = irrgen.front_values(8, n1 + 31 * n2, n1 + n2)
    F11, F12, F21, F22 = F[:n1, :n1], F[:n1, n1:], F[n1:, :n1], F[n1:, n1:]
    o11, o12, o22, ipiv, info = orc.getrf_partial(F11, F12, F21, F22)
    if n1 == 0:
        assert np.array_equal(o22, F22)
        return
    LU, ip, inf2, _ = orc.getrf(F11)
    assert np.array_equal(o11, LU) and np.array_equal(ipiv, ip)
    if n2 == 0:
        return
    X = sl.solve(F11, F12)
    S = F22 - F21 @ X
    assert np.abs(o12 - X).max() <= 1e-10 * max(1, np.abs(X).max())
    assert np.abs(o22 - S).max() <= 1e-10 * max(1, np.abs(S).max())


def test_partial_batch_equals_single(orc):
    rng = np.random.default_rng(0)
    fronts, refs = [], []
    for i in range(12):
        n1, n2 = int(rng.integers(0, 20)), int(rng.integers(0, 20))
        F = irrgen.front_values(3, i, n1 + n2)
        fr = dict(F11=F[:n1, :n1].copy(order="F"), F12=F[:n1, n1:].copy(order="F"),
                  F21=F[n1:, :n1].copy(order="F"), F22=F[n1:, n1:].copy(order="F"))
        refs.append(orc.getrf_partial(fr["F11"], fr["F12"], fr["F21"], fr["F22"]))
        fronts.append(fr)
    ipivs, info = orc.getrf_partial_batch(fronts, nthreads=3)
    for fr, r, p, inf in zip(fronts, refs, ipivs, info):
        assert np.array_equal(fr["F11"], r[0]) and np.array_equal(fr["F12"], r[1])
        assert np.array_equal(fr["F22"], r[2]) and np.array_equal(p, r[3]) and inf == r[4]


# ---------------------------------------------------------------- building blocks
def test_gemm_integer_exact(orc):
    rng = np.random.default_rng(1)
    for ta, tb in itertools.product((0, 1), repeat=2):
        m, n, k = 7, 5, 9
        A = rng.integers(-5, 6, size=(k, m) if ta else (m, k)).astype(float)
        B = rng.integers(-5, 6, size=(n, k) if tb else (k, n)).astype(float)
        Cm = rng.integers(-5, 6, size=(m, n)).astype(float)
        out = orc.gemm(ta, tb, -1.0, A, B, 2.0, Cm)
        ref = -1.0 * ((A.T if ta else A) @ (B.T if tb else B)) + 2.0 * Cm
        assert np.array_equal(out, ref)
    nanC = np.full((3, 3), np.nan)
    out = orc.gemm(0, 0, 1.0, np.eye(3), np.eye(3), 0.0, nanC)   # beta = 0 ignores C
    assert np.array_equal(out, np.eye(3))


@pytest.mark.parametrize("side,uplo,trans,diag", list(itertools.product((0, 1), repeat=4)))
def test_trsm_recovers_dyadic_solution(orc, side, uplo, trans, diag):
    """B = op(T) X0 (left) or X0 op(T) (right) with dyadic T, integer X0:
    the solve recovers X0 exactly (all 16 BLAS combinations)."""
    rng = np.random.default_rng(side * 8 + uplo * 4 + trans * 2 + diag)
    m, n = 6, 4
    kt = n if side else m
    T = rng.integers(-4, 5, size=(kt, kt)).astype(float) / 4.0
    np.fill_diagonal(T, rng.choice([1.0, -1.0, 2.0, -2.0], size=kt))
    Tf = np.triu(T) if uplo else np.tril(T)
    if diag:
        np.fill_diagonal(Tf, 1.0)
    opT = Tf.T if trans else Tf
    X0 = rng.integers(-6, 7, size=(m, n)).astype(float)
    B = (X0 @ opT) if side else (opT @ X0)
    T_junk = T.copy()                        # the other triangle must not be read
    if uplo:
        T_junk[np.tril_indices(kt, -1)] = 1e300
    else:
        T_junk[np.triu_indices(kt, 1)] = 1e300
    if diag:
        np.fill_diagonal(T_junk, 1e300)
    X = orc.trsm(side, uplo, trans, diag, 2.0, T_junk, B / 2.0)
    assert np.array_equal(X, X0)


def test_laswp(orc):
    A = irrgen.uniform_values(1, 3, 6, 4)
    assert np.array_equal(orc.laswp(A, 0, 4, np.array([1, 2, 3, 4])), A)
    piv = np.array([3, 5, 3, 6])
    out = orc.laswp(A, 0, 4, piv)
    assert np.array_equal(out, apply_swaps(A, piv))
    # undo: applying the swaps in reverse order restores A
    back = out.copy()
    for k in range(3, -1, -1):
        back = orc.laswp(back, k, k + 1, piv)
    assert np.array_equal(back, A)
    # partial ranges
    assert np.array_equal(orc.laswp(A, 1, 3, piv), apply_swaps(A, [1, 5, 3, 4]))


# ---------------------------------------------------------------- flop formula
def count_gepp_ops(m, n):
    """Operations actually performed by unblocked GEPP with one reciprocal
    per column (LAPACK dgetf2): the count FLOPS_DGETRF models."""
    ops = 0
    for k in range(min(m, n)):
        r = m - k - 1
        ops += 1 + r + 2 * r * (n - k - 1)
    return ops


def test_flops_formula():
    from paper_conf_sc_abdelfattahgbtld22_b200 import flops
    for m in range(0, 40):
        for n in range(0, 40):
            # m >= n: the count of the operations GEPP performs; m < n: SURVEY Q1
            # (LAPACK/MAGMA FLOPS_DGETRF) counts the transposed problem.
            ref = count_gepp_ops(m, n) if m >= n else count_gepp_ops(n, m)
            assert flops.getrf_flops(m, n) == pytest.approx(ref, abs=1e-6)
    assert flops.getrf_flops(1, 1) == 1.0
    # partial: getrf(n1) + two triangular solves n1^2 n2 each + Schur GEMM 2 n1 n2^2
    assert flops.partial_flops(3, 2) == pytest.approx(count_gepp_ops(3, 3) + 2 * 9 * 2 + 2 * 3 * 4)


# ---------------------------------------------------------------- GETRS pins
def test_getrs_hand_2x2(orc):
    """A = [[1, 2], [3, 4]]: GEPP swaps rows (ipiv = [2, 2]), L = [[1,0],[1/3,1]],
    U = [[3, 4], [0, 2/3]]; A x = [5, 11] has x = [1, 2] (worked by hand)."""
    A = np.array([[1.0, 2.0], [3.0, 4.0]], order="F")
    LU, ipiv, info, _ = orc.getrf(A)
    assert list(ipiv) == [2, 2] and info == 0
    X = orc.getrs(LU, ipiv, np.array([[5.0], [11.0]], order="F"))
    assert np.abs(X[:, 0] - [1.0, 2.0]).max() <= 4 * EPS


@pytest.mark.parametrize("n,nrhs", [(1, 1), (5, 3), (17, 1), (40, 9), (64, 64)])
def test_getrs_exact_dyadic(orc, n, nrhs):
    """G1: A = P L U from dyadic factors with power-of-two pivots, X dyadic,
    B = A X formed exactly (integers scaled by powers of two) -> GETRS returns X
    bit-exactly (every step of the solve is exact on this family)."""
    A, L, U, ipiv, info = irrgen.g1_exact(9, n + 13 * nrhs, n, n)
    rng = np.random.default_rng(n * 100 + nrhs)
    X = np.asfortranarray(rng.integers(-8, 9, size=(n, nrhs)).astype(np.float64))
    B = np.asfortranarray(A @ X)
    LU, oipiv, _, _ = orc.getrf(A)
    assert np.array_equal(oipiv, ipiv)
    got = orc.getrs(LU, oipiv, B)
    assert np.array_equal(got, X)


@pytest.mark.parametrize("n,nrhs", [(3, 2), (33, 5), (100, 17)])
def test_getrs_vs_lapack(orc, n, nrhs):
    """Cross-check against LAPACK dgetrs (scipy lu_solve on the oracle's own
    factors): same factors in, same solution out to rounding."""
    A = irrgen.uniform_values(12, n, n, n)
    B = irrgen.uniform_values(13, n, n, nrhs)
    LU, ipiv, _, _ = orc.getrf(A)
    got = orc.getrs(LU, ipiv, B)
    ref = sl.lu_solve((LU, ipiv - 1), B)
    assert np.abs(got - ref).max() <= 1e-9 * max(1.0, np.abs(ref).max())
    res = np.abs(A @ got - B).max() / (np.abs(A).max() * np.abs(got).max() * n * EPS)
    assert res <= 10.0

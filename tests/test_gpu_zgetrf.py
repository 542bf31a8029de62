"""GPU parity of irr_zgetrf (complex LU with partial pivoting, SURVEY §8(f)
NEXT 3; the solver's A in C^{N x N}) through the C ABI against
oracle.zgetrf (LAPACK zgetf2 semantics, izamax pivoting):
  * the exact complex dyadic family zG1: L, U, ipiv bit-exact (construction);
  * zG1-singular: info = c + 1, exact factors;
  * uniform complex values: ipiv / info equal where the oracle's pivots are
    well separated, backward error <= 10 (complex Frobenius norm, Q11), L / U
    within 1e-10 normwise-max relative (Q12);
  * bad per-matrix arguments skipped with info < 0.
Sizes cover the shared-memory path (m n <= 4096) and the global path, ld > m,
tall / wide / ragged panels (nb = 16)."""
import numpy as np
import pytest

import irrgen
import oracle

pytestmark = pytest.mark.gpu

torch = pytest.importorskip("torch")
if not torch.cuda.is_available():
    pytest.skip("no CUDA device", allow_module_level=True)

from gpu_util import rel_dev  # noqa: E402
from paper_conf_sc_abdelfattahgbtld22_b200.batch import ZMatrixBatch  # noqa: E402

NEAR_TIE = 1.0 + 1e-6


def _zgetrf(mats, ld_extra=0, m=None):
    ma = [A.shape[0] for A in mats]
    na = [A.shape[1] for A in mats]
    B = ZMatrixBatch(ma, na, [max(1, a + ld_extra) for a in ma])
    if m is not None:
        B.m = torch.tensor(m, dtype=torch.int32, device="cuda")
    host = np.full(B.total, np.nan)
    for i, A in enumerate(mats):
        if A.size:
            B.matrix(i, host)[:, :] = A
    B.data.copy_(torch.from_numpy(host))
    B.getrf()
    torch.cuda.synchronize()
    out, ip = B.data.cpu().numpy(), B.ipiv_data.cpu().numpy()
    info = B.info.cpu().numpy()[: B.batch]
    return [np.array(B.matrix(i, out)) for i in range(B.batch)], [np.array(B.ipiv_of(i, ip)) for i in
                                                                   range(B.batch)], info


SHAPES = [(1, 1), (7, 7), (16, 16), (17, 9), (9, 17), (33, 33), (64, 64), (65, 63), (100, 41), (41, 100),
          (150, 150), (300, 200), (200, 300), (513, 513)]


@pytest.mark.parametrize("ld_extra", [0, 3])
def test_zg1_exact(ld_extra):
    mats, refs = [], []
    for g, (m, n) in enumerate(SHAPES):
        A, L, U, ipiv, _ = irrgen.zg1_exact(50, g, m, n)
        mats.append(A)
        refs.append((L, U, ipiv))
    LUs, ipivs, info = _zgetrf(mats, ld_extra)
    for (m, n), LU, ip, inf, (L, U, ipiv) in zip(SHAPES, LUs, ipivs, info, refs):
        k = min(m, n)
        assert inf == 0 and np.array_equal(ip, ipiv), (m, n)
        assert np.array_equal(np.tril(LU[:, :k], -1) + np.eye(m, k), L), (m, n)
        assert np.array_equal(np.triu(LU[:k, :]), U), (m, n)


def test_zg1_singular():
    cases = [(6, 6, 0), (40, 40, 17), (90, 90, 89), (300, 300, 150)]
    mats = [irrgen.zg1_exact(51, g, m, n, singular_col=c)[0] for g, (m, n, c) in enumerate(cases)]
    LUs, ipivs, info = _zgetrf(mats)
    for (m, n, c), A, LU, ip, inf in zip(cases, mats, LUs, ipivs, info):
        LUo, ipo, info_o, _ = oracle.zgetrf(A)
        assert inf == info_o == c + 1 and np.array_equal(ip, ipo)
        assert np.array_equal(LU, LUo)


def test_uniform_vs_oracle():
    rng = np.random.default_rng(52)
    shapes = SHAPES + [(int(a), int(b)) for a, b in zip(rng.integers(1, 300, 40), rng.integers(1, 300, 40))]
    mats = [irrgen.zuniform_values(53, g, m, n) for g, (m, n) in enumerate(shapes)]
    LUs, ipivs, info = _zgetrf(mats)
    ties = 0
    for g, (A, LU, ip, inf) in enumerate(zip(mats, LUs, ipivs, info)):
        LUo, ipo, info_o, sep = oracle.zgetrf(A)
        be = oracle.zbackward_error(A, LU, ip)
        assert be <= 10.0, (g, A.shape, be)
        k = min(A.shape)
        # the GPU's pivots are izamax choices in its own arithmetic: every
        # step-k candidate l_rk u_kk has |Re| + |Im| <= that of u_kk (G8)
        Lk = np.tril(LU[:, :k], -1) * np.diag(LU)[None, :k]
        c1 = np.abs(Lk.real) + np.abs(Lk.imag)
        d1 = np.abs(np.diag(LU)[:k].real) + np.abs(np.diag(LU)[:k].imag)
        assert np.all(c1 <= d1[None, :] * (1 + 1e-14)), (g, A.shape)
        if np.array_equal(ip, ipo):
            assert inf == info_o
            L, Lo = np.tril(LU[:, :k], -1), np.tril(LUo[:, :k], -1)
            U, Uo = np.triu(LU[:k, :]), np.triu(LUo[:k, :])
            assert rel_dev(L, Lo) <= 1e-10 and rel_dev(U, Uo) <= 1e-10, (g, A.shape)
        else:
            assert sep < NEAR_TIE, (g, A.shape, sep)
            ties += 1
    assert ties <= 2


def test_bad_arguments_are_skipped():
    mats = [irrgen.zuniform_values(54, g, s, s) for g, s in enumerate((10, 20, 30))]
    LUs, ipivs, info = _zgetrf(mats, m=[10, -2, 30])
    assert info[1] == -1 and info[0] == 0 and info[2] == 0
    for g in (0, 2):
        LUo, ipo, _, _ = oracle.zgetrf(mats[g])
        assert np.array_equal(ipivs[g], ipo)

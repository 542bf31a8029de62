"""The few-large regime (§V-A, Fig. 11: the
crossover against cuSOLVER at ~5k): matrices and partial fronts of 4096-8192,
alone and mixed with small ones, through the grid-wide tier (windowed panels
of 512 / 1024 threads above 2048 rows, pivot ranges above 4096 applied in
pieces).  The exact families are checked against their construction (an
oracle GEPP of an 8192^2 matrix is minutes of single-core time); one uniform
4096^2 matrix is checked against the oracle (marked `full`)."""
import numpy as np
import pytest

import irrgen

pytestmark = pytest.mark.gpu

torch = pytest.importorskip("torch")
if not torch.cuda.is_available():
    pytest.skip("no CUDA device", allow_module_level=True)

from gpu_util import check_getrf, gpu_getrf, gpu_partial  # noqa: E402
from paper_conf_sc_abdelfattahgbtld22_b200 import irr  # noqa: E402


@pytest.fixture(autouse=True)
def _reset_tuning():
    irr.irr_reset_tuning()
    yield
    irr.irr_reset_tuning()


@pytest.mark.parametrize("nbo,split", [(0, 0), (128, 0), (128, 1)])
def test_large_g1_exact(nbo, split):
    """split = 1: the two-level inner steps' trailing update as a grid-wide
    GEMM (tuning split_strip, the few-large path)."""
    irr.irr_set_tuning("nb_outer", nbo)
    irr.irr_set_tuning("split_strip", split)
    shapes = [(4096, 4096), (5000, 3000), (3000, 5000), (8192, 700), (40, 40), (300, 300)]
    mats = [irrgen.g1_exact(61, g, m, n)[0] for g, (m, n) in enumerate(shapes)]
    refs = [irrgen.g1_exact(61, g, m, n) for g, (m, n) in enumerate(shapes)]
    LUs, ipivs, info, _ = gpu_getrf(mats)
    for (m, n), LU, ip, inf, (_, L, U, ipiv, _) in zip(shapes, LUs, ipivs, info, refs):
        k = min(m, n)
        assert inf == 0 and np.array_equal(ip, ipiv), (m, n)
        assert np.array_equal(np.tril(LU[:, :k], -1) + np.eye(m, k), L), (m, n)
        assert np.array_equal(np.triu(LU[:k, :]), U), (m, n)


def test_large_8192_exact():
    A, L, U, ipiv, _ = irrgen.g1_exact(62, 0, 8192, 8192)
    LUs, ipivs, info, _ = gpu_getrf([A])
    assert info[0] == 0 and np.array_equal(ipivs[0], ipiv)
    assert np.array_equal(np.tril(LUs[0], -1) + np.eye(8192), L)
    assert np.array_equal(np.triu(LUs[0]), U)


@pytest.mark.parametrize("n1,n2", [(4500, 1500), (6000, 300)])
def test_large_partial_front_exact(n1, n2):
    """G1' fronts with n1 > 4096 (fused a5.2 above its 4096 limit -> LASWP in
    pieces + 2 x TRSM): F12 -> X, F22 -> S bit-exactly."""
    f = irrgen.g1_front(63, n1, n1, n2)
    F = np.zeros((n1 + n2, n1 + n2), order="F")
    F[:n1, :n1], F[:n1, n1:], F[n1:, :n1], F[n1:, n1:] = f["F11"], f["F12"], f["F21"], f["F22"]
    out, ipivs, info = gpu_partial([(F, n1), (irrgen.front_values(64, 1, 50), 20)])
    assert info[0] == 0 and np.array_equal(ipivs[0], f["ipiv"])
    assert np.array_equal(out[0][:n1, n1:], f["X"])
    assert np.array_equal(out[0][n1:, n1:], f["S"])


@pytest.mark.full
def test_large_uniform_vs_oracle():
    A = irrgen.uniform_values(65, 0, 4096, 4096)
    B = irrgen.uniform_values(65, 1, 4500, 2000)
    LUs, ipivs, info, _ = gpu_getrf([A, B])
    for M, LU, ip, inf in zip((A, B), LUs, ipivs, info):
        assert check_getrf(M, LU, ip, int(inf), label=str(M.shape)) in ("match", "near-tie")

"""GPU parity of irr_getrf_partial (LU(F11), F12 <- U^-1 L^-1 P^T F12,
F22 <- F22 - F21 F12, F21 untouched) against the oracle."""
import numpy as np
import pytest

import irrgen

pytestmark = pytest.mark.gpu

torch = pytest.importorskip("torch")
if not torch.cuda.is_available():
    pytest.skip("no CUDA device", allow_module_level=True)

from gpu_util import check_partial, gpu_partial  # noqa: E402
from paper_conf_sc_abdelfattahgbtld22_b200 import irr  # noqa: E402


@pytest.fixture(autouse=True)
def _reset_tuning():
    irr.irr_reset_tuning()
    yield
    irr.irr_reset_tuning()


def _g1_front(seed, gid, n1, n2):
    f = irrgen.g1_front(seed, gid, n1, n2)
    F = np.zeros((n1 + n2, n1 + n2), order="F")
    F[:n1, :n1], F[:n1, n1:], F[n1:, :n1], F[n1:, n1:] = f["F11"], f["F12"], f["F21"], f["F22"]
    return F, f


SHAPES = [(1, 1), (5, 7), (16, 3), (31, 1), (32, 40), (33, 65), (64, 200), (120, 40), (150, 150), (300, 600),
          (700, 300)]


@pytest.mark.parametrize("tier", ["default", "L", "unfused"])
def test_g1_front_exact(tier):
    """G1': F12 -> X, F22 -> S bit-exactly, F11 -> the chosen L\\U.  "unfused":
    step a5.2 as irrLASWP + 2 x irrTRSM instead of the fused strip kernel."""
    if tier == "unfused":
        irr.irr_set_tuning("getrs_fused", 0)
    if tier == "L":
        irr.irr_set_tuning("tier_s", 0)
        irr.irr_set_tuning("tier_m_max", 0)
    fronts, refs = [], []
    for g, (n1, n2) in enumerate(SHAPES):
        F, f = _g1_front(21, g, n1, n2)
        fronts.append((F, n1))
        refs.append(f)
    out, ipivs, info = gpu_partial(fronts)
    for (F, n1), Fg, ip, inf, f in zip(fronts, out, ipivs, info, refs):
        assert inf == 0 and np.array_equal(ip, f["ipiv"])
        assert np.array_equal(Fg[:n1, n1:], f["X"]), (n1, F.shape)
        assert np.array_equal(Fg[n1:, n1:], f["S"]), (n1, F.shape)
        check_partial(F, n1, Fg, ip, int(inf), exact=True, label=f"{n1}/{F.shape[0]}")


@pytest.mark.parametrize("fused", [1, 0])
def test_uniform_fronts_vs_oracle(fused):
    irr.irr_set_tuning("getrs_fused", fused)
    shapes = [(1, 0), (7, 0), (3, 4), (10, 10), (17, 40), (50, 80), (97, 31), (129, 257), (400, 500)]
    fronts = [(irrgen.front_values(8, g, n1 + n2), n1) for g, (n1, n2) in enumerate(shapes)]
    out, ipivs, info = gpu_partial(fronts)
    for g, ((F, n1), Fg, ip, inf) in enumerate(zip(fronts, out, ipivs, info)):
        check_partial(F, n1, Fg, ip, int(inf), label=f"front {g}")


def test_c4_shaped_sample():
    """configs[3] size rule (heavy tail) on a bounded sample incl. a 3k-4k front."""
    cfg = irrgen.config("C4", scale=0.004)            # 200 fronts
    n1 = list(cfg.m) + [1200]
    n2 = list(cfg.n) + [2100]
    fronts = [(irrgen.front_values(cfg.seed, g, int(a + b)), int(a)) for g, (a, b) in enumerate(zip(n1, n2))]
    out, ipivs, info = gpu_partial(fronts)
    st = {}
    for g, ((F, a), Fg, ip, inf) in enumerate(zip(fronts, out, ipivs, info)):
        r = check_partial(F, a, Fg, ip, int(inf), label=f"C4 {g}")
        st[r] = st.get(r, 0) + 1
    assert st.get("match", 0) >= len(fronts) - 2


LAPACK_SHAPES = [(1, 1), (5, 7), (16, 3), (31, 1), (32, 40), (33, 65), (64, 200), (120, 40), (150, 150),
                 (300, 200), (3, 0), (0, 5)]


@pytest.mark.parametrize("tier", ["default", "L", "unfused"])
def test_lapack_partial_exact(tier):
    """G1'' fronts through irr_getrf_partial_lapack:
    F12 -> U12 = X, F21 -> L21 = Y, F22 -> S, F11 -> the chosen L\\U, all
    bit-exact (the construction, no oracle needed).  "unfused": U12 through
    irrLASWP + irrTRSM instead of the strip kernel stopped before U^-1."""
    if tier == "unfused":
        irr.irr_set_tuning("getrs_fused", 0)
    if tier == "L":
        irr.irr_set_tuning("tier_s", 0)
        irr.irr_set_tuning("tier_m_max", 0)
    fronts, refs = [], []
    for g, (n1, n2) in enumerate(LAPACK_SHAPES):
        f = irrgen.g1_front_lapack(23, g, n1, n2)
        F = np.zeros((n1 + n2, n1 + n2), order="F")
        F[:n1, :n1], F[:n1, n1:], F[n1:, :n1], F[n1:, n1:] = f["F11"], f["F12"], f["F21"], f["F22"]
        fronts.append((F, n1))
        refs.append(f)
    out, ipivs, info = gpu_partial(fronts, lapack=True)
    for (F, n1), Fg, ip, inf, f in zip(fronts, out, ipivs, info, refs):
        assert inf == 0 and np.array_equal(ip, f["ipiv"]), (n1, F.shape)
        assert np.array_equal(Fg[:n1, :n1], np.tril(f["L"], -1) + f["U"]), (n1, F.shape)
        assert np.array_equal(Fg[:n1, n1:], f["X"]), (n1, F.shape)
        assert np.array_equal(Fg[n1:, :n1], f["Y"]), (n1, F.shape)
        assert np.array_equal(Fg[n1:, n1:], f["S"]), (n1, F.shape)


@pytest.mark.parametrize("fused", [1, 0])
def test_lapack_partial_vs_oracle(fused):
    """Uniform fronts against oracle.getrf_partial_lapack: ipiv / info equal
    (well-separated pivots), F11 / U12 / L21 within 1e-10 normwise-max
    relative, F22 within 1e-10 of sigma = max(|F22_in| + |L21_o| |U12_o|)."""
    from gpu_util import rel_dev
    import oracle
    irr.irr_set_tuning("getrs_fused", fused)
    shapes = [(1, 0), (7, 0), (3, 4), (10, 10), (17, 40), (50, 80), (97, 31), (129, 257), (400, 500), (33, 700)]
    fronts = [(irrgen.front_values(88, g, n1 + n2), n1) for g, (n1, n2) in enumerate(shapes)]
    out, ipivs, info = gpu_partial(fronts, lapack=True)
    for g, ((F, a), Fg, ip, inf) in enumerate(zip(fronts, out, ipivs, info)):
        o11, o12, o21, o22, ipo, info_o = oracle.getrf_partial_lapack(F[:a, :a], F[:a, a:], F[a:, :a], F[a:, a:])
        assert inf == info_o and np.array_equal(ip, ipo), g
        for got, want in ((Fg[:a, :a], o11), (Fg[:a, a:], o12), (Fg[a:, :a], o21)):
            assert rel_dev(got, want) <= 1e-10, g
        if o22.size:
            sigma = (np.abs(F[a:, a:]) + np.abs(o21) @ np.abs(o12)).max()
            assert np.abs(Fg[a:, a:] - o22).max() <= 1e-10 * sigma, g

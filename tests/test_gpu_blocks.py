"""GPU parity of the exported building blocks irr_gemm / irr_trsm / irr_laswp
 with the expanded interface and DCWI clamps, against the oracle.
Integer / dyadic data make every expected value exact."""
import itertools

import numpy as np
import pytest

pytestmark = pytest.mark.gpu

torch = pytest.importorskip("torch")
if not torch.cuda.is_available():
    pytest.skip("no CUDA device", allow_module_level=True)

import oracle  # noqa: E402
from paper_conf_sc_abdelfattahgbtld22_b200 import irr  # noqa: E402
from paper_conf_sc_abdelfattahgbtld22_b200.batch import MatrixBatch  # noqa: E402


@pytest.fixture(autouse=True)
def _reset_tuning():
    yield
    irr.irr_reset_tuning()


def _upload(mats):
    B = MatrixBatch([a.shape[0] for a in mats], [a.shape[1] for a in mats], with_ipiv=False)
    host = np.zeros(B.total)
    for i, a in enumerate(mats):
        if a.size:
            B.matrix(i, host)[:, :] = a
    B.data.copy_(torch.from_numpy(host))
    return B


def _download(B):
    out = B.data.cpu().numpy()
    return [np.array(B.matrix(i, out)) for i in range(B.batch)]


def _i32(x):
    return torch.tensor(np.asarray(x, dtype=np.int32), device="cuda")


@pytest.mark.parametrize("ta,tb,use_work", list(itertools.product((0, 1), (0, 1), (True, False))))
def test_gemm_dcwi_exact(ta, tb, use_work):
    rng = np.random.default_rng(ta * 4 + tb * 2 + use_work)
    batch = 9
    m = rng.integers(1, 150, batch); n = rng.integers(1, 150, batch); k = rng.integers(1, 90, batch)
    m[0], n[0], k[0] = 0, 5, 5          # empty
    Ai, Aj, Bi, Bj, Ci, Cj = 3, 2, 1, 4, 2, 5
    M, N, K = 120, 130, 70               # required dims (clamped per matrix)
    As = [rng.integers(-4, 5, size=(k[i], m[i]) if ta else (m[i], k[i])).astype(float) for i in range(batch)]
    Bs = [rng.integers(-4, 5, size=(n[i], k[i]) if tb else (k[i], n[i])).astype(float) for i in range(batch)]
    Cs = [rng.integers(-4, 5, size=(m[i], n[i])).astype(float) for i in range(batch)]
    dA, dB, dC = _upload(As), _upload(Bs), _upload(Cs)
    work = torch.empty(irr.irr_gemm_workspace_size(batch), dtype=torch.uint8, device="cuda") if use_work else None
    irr.irr_gemm(ta, tb, M, N, K, _i32(m), _i32(n), _i32(k), -1.0, dA.ptr, Ai, Aj, dA.ld, dB.ptr, Bi, Bj, dB.ld,
                 2.0, dC.ptr, Ci, Cj, dC.ld, batch, work=work)
    torch.cuda.synchronize()
    got = _download(dC)
    for i in range(batch):
        a_m_off, a_k_off = (Aj, Ai) if ta else (Ai, Aj)
        b_k_off, b_n_off = (Bj, Bi) if tb else (Bi, Bj)
        me = min(M, m[i] - a_m_off, m[i] - Ci)
        ne = min(N, n[i] - b_n_off, n[i] - Cj)
        ke = max(0, min(K, k[i] - a_k_off, k[i] - b_k_off))
        exp = Cs[i].copy()
        if me > 0 and ne > 0:
            Asub = As[i][Ai:Ai + (ke if ta else me), Aj:Aj + (me if ta else ke)]
            Bsub = Bs[i][Bi:Bi + (ne if tb else ke), Bj:Bj + (ke if tb else ne)]
            Csub = exp[Ci:Ci + me, Cj:Cj + ne]
            exp[Ci:Ci + me, Cj:Cj + ne] = oracle.gemm(ta, tb, -1.0, Asub, Bsub, 2.0, Csub)
        assert np.array_equal(got[i], exp), i


@pytest.mark.parametrize("warps", [8, 9])
@pytest.mark.parametrize("ta,tb", list(itertools.product((0, 1), (0, 1))))
def test_gemm_big_core_exact(ta, tb, warps):
    """Products large enough for the 128 x 128 DMMA core (several tiles, ragged
    edges, K not a multiple of the 16-chunk) mixed with small ones that stay
    on the 64 x 64 core; integer data, so every entry is exact.  warps = 9:
    the warp-specialised core (producer warp + mbarrier ring)."""
    irr.irr_set_tuning("xgemm_warps", warps)
    rng = np.random.default_rng(100 + ta * 2 + tb)
    m = np.array([300, 97, 5, 260, 130, 64]); n = np.array([257, 140, 200, 96, 7, 64])
    k = np.array([201, 48, 300, 77, 130, 40])
    batch = len(m)
    As = [rng.integers(-4, 5, size=(k[i], m[i]) if ta else (m[i], k[i])).astype(float) for i in range(batch)]
    Bs = [rng.integers(-4, 5, size=(n[i], k[i]) if tb else (k[i], n[i])).astype(float) for i in range(batch)]
    Cs = [rng.integers(-4, 5, size=(m[i], n[i])).astype(float) for i in range(batch)]
    dA, dB, dC = _upload(As), _upload(Bs), _upload(Cs)
    work = torch.empty(irr.irr_gemm_workspace_size(batch), dtype=torch.uint8, device="cuda")
    irr.irr_gemm(ta, tb, int(m.max()), int(n.max()), int(k.max()), _i32(m), _i32(n), _i32(k), -1.0, dA.ptr, 0, 0,
                 dA.ld, dB.ptr, 0, 0, dB.ld, 0.5, dC.ptr, 0, 0, dC.ld, batch, work=work)
    torch.cuda.synchronize()
    got = _download(dC)
    for i in range(batch):
        exp = oracle.gemm(ta, tb, -1.0, As[i], Bs[i], 0.5, Cs[i])
        assert np.array_equal(got[i], exp), i


@pytest.mark.parametrize("side,uplo,trans,diag", list(itertools.product((0, 1), repeat=4)))
def test_trsm_all_combinations_exact(side, uplo, trans, diag):
    """B = op(T) X0 (left) or X0 op(T) (right), dyadic T, integer X0: the
    recursive solve (leaf 8 here, so several levels) recovers X0 exactly."""
    irr.irr_set_tuning("trsm_nb", 8)
    try:
        rng = np.random.default_rng(side * 8 + uplo * 4 + trans * 2 + diag)
        batch = 5
        ms = [1, 9, 40, 70, 0]
        ns = [3, 17, 33, 50, 4]
        Ts, Bs, X0s = [], [], []
        for i in range(batch):
            kt = ns[i] if side else ms[i]
            T = rng.integers(-2, 3, size=(kt, kt)).astype(float) / 8.0
            np.fill_diagonal(T, rng.choice([1.0, -1.0, 2.0, -2.0], size=kt))
            Tf = np.triu(T) if uplo else np.tril(T)
            if diag:
                np.fill_diagonal(Tf, 1.0)
            opT = Tf.T if trans else Tf
            X0 = rng.integers(-3, 4, size=(ms[i], ns[i])).astype(float)
            B = (X0 @ opT) if side else (opT @ X0)
            Tj = T.copy()
            if uplo:
                Tj[np.tril_indices(kt, -1)] = 1e300
            else:
                Tj[np.triu_indices(kt, 1)] = 1e300
            if diag:
                np.fill_diagonal(Tj, 1e300)
            Ts.append(Tj); Bs.append(B * 0.5); X0s.append(X0)
        dT, dB = _upload(Ts), _upload(Bs)
        work = torch.empty(irr.irr_trsm_workspace_size(batch), dtype=torch.uint8, device="cuda")
        irr.irr_trsm(side, uplo, trans, diag, max(ms), max(ns), _i32(ms), _i32(ns), 2.0, dT.ptr, 0, 0, dT.ld,
                     dB.ptr, 0, 0, dB.ld, batch, work=work)
        torch.cuda.synchronize()
        got = _download(dB)
        for i in range(batch):
            assert np.array_equal(got[i], X0s[i]), (i, np.abs(got[i] - X0s[i]).max() if got[i].size else 0)
    finally:
        irr.irr_reset_tuning()


def test_trsm_offsets_match_oracle():
    rng = np.random.default_rng(5)
    Ts = [np.tril(rng.standard_normal((60, 60))) + 8 * np.eye(60), np.tril(rng.standard_normal((30, 30))) + 8 * np.eye(30)]
    Bs = [rng.standard_normal((60, 20)), rng.standard_normal((30, 9))]
    dT, dB = _upload(Ts), _upload(Bs)
    ms, ns = [60, 30], [20, 9]
    irr.irr_trsm(0, 0, 0, 0, 40, 15, _i32(ms), _i32(ns), 1.0, dT.ptr, 10, 10, dT.ld, dB.ptr, 10, 2, dB.ld, 2)
    torch.cuda.synchronize()
    got = _download(dB)
    for i in range(2):
        me = min(40, ms[i] - 10)
        ne = min(15, ns[i] - 2)
        exp = Bs[i].copy()
        exp[10:10 + me, 2:2 + ne] = oracle.trsm(0, 0, 0, 0, 1.0, Ts[i][10:10 + me, 10:10 + me], exp[10:10 + me, 2:2 + ne])
        assert np.abs(got[i] - exp).max() <= 1e-13 * np.abs(exp).max()


def test_laswp_matches_oracle():
    rng = np.random.default_rng(3)
    batch = 4
    ms, ns = [10, 50, 300, 7], [6, 40, 100, 3]
    mats = [rng.standard_normal((ms[i], ns[i])) for i in range(batch)]
    kc = [8, 45, 290, 0]
    ipivs = []
    for i in range(batch):
        ip = np.array([k + 1 + rng.integers(0, ms[i] - k) for k in range(kc[i])], dtype=np.int32)
        ipivs.append(ip)
    dA = _upload(mats)
    ipflat = torch.tensor(np.concatenate([p for p in ipivs] + [np.zeros(1, np.int32)]), device="cuda")
    offs = np.concatenate([[0], np.cumsum([len(p) for p in ipivs])[:-1]])
    iptr = torch.tensor(ipflat.data_ptr() + 4 * offs, dtype=torch.int64, device="cuda")
    k1, k2 = 2, 200
    irr.irr_laswp(60, _i32(ns), dA.ptr, 0, 1, dA.ld, k1, k2, _i32(kc), iptr, batch)
    torch.cuda.synchronize()
    got = _download(dA)
    for i in range(batch):
        exp = mats[i].copy()
        kend = min(k2, kc[i])
        if kend > k1:
            exp[:, 1:1 + min(60, ns[i] - 1)] = oracle.laswp(exp[:, 1:1 + min(60, ns[i] - 1)], k1, kend, ipivs[i])
        assert np.array_equal(got[i], exp), i

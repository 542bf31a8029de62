"""GPU parity of irr_getrf (through the C ABI) against the CPU oracle.

Covers every tier (S: warp per matrix, M: CTA with the matrix in shared
memory, L: blocked right-looking with panel / swap+TRSM / GEMM kernels), the
size edge cases of SURVEY §8(c) ("Sizes the unit tests must cover"), ld > m,
bad arguments, exact families (bit-exact) and the configs of BASELINE.json.
"""
import numpy as np
import pytest

import irrgen

pytestmark = pytest.mark.gpu

torch = pytest.importorskip("torch")
if not torch.cuda.is_available():
    pytest.skip("no CUDA device", allow_module_level=True)

from gpu_util import check_getrf, gpu_getrf  # noqa: E402
from paper_conf_sc_abdelfattahgbtld22_b200 import irr  # noqa: E402


@pytest.fixture(autouse=True)
def _reset_tuning():
    irr.irr_reset_tuning()
    yield
    irr.irr_reset_tuning()


EDGE = [0, 1, 2, 3, 7, 8, 15, 16, 17, 31, 32, 33, 63, 64, 65, 127, 128, 129]


def _uniform(shapes, seed=77):
    return [irrgen.uniform_values(seed, g, m, n) for g, (m, n) in enumerate(shapes)]


def _run_and_check(mats, exact=False, **kw):
    LUs, ipivs, info, _ = gpu_getrf(mats, **kw)
    stats = {}
    for g, (A, LU, ip, inf) in enumerate(zip(mats, LUs, ipivs, info)):
        st = check_getrf(A, LU, ip, int(inf), exact=exact, label=f"#{g} {A.shape}")
        stats[st] = stats.get(st, 0) + 1
    return stats


def test_c1_parity():
    """configs[0]: 100 square matrices n ~ U{1..32} (tier S)."""
    cfg = irrgen.config("C1")
    mats = [irrgen.uniform_values(cfg.seed, g, int(m), int(n)) for g, (m, n) in enumerate(zip(cfg.m, cfg.n))]
    st = _run_and_check(mats)
    assert st.get("match", 0) >= 98


def test_edge_shapes_all_tiers():
    shapes = [(m, n) for m in EDGE for n in EDGE]
    st = _run_and_check(_uniform(shapes))
    assert st.get("match", 0) + st.get("empty", 0) >= len(shapes) - 2


@pytest.mark.parametrize("mid_dmma", [0, 1])
@pytest.mark.parametrize("tier_m_max", [None, 12288, 24576])
def test_tier_m_boundary_and_extreme_shapes(tier_m_max, mid_dmma):
    # m * n around the tier-M limits (48 / 96 / 192 KB footprints) and very
    # thin shapes, at the default limit and with the two larger bins enabled;
    # mid_dmma = 1: the in-shared-memory trailing update on the DMMA core
    if tier_m_max is not None:
        irr.irr_set_tuning("tier_m_max", tier_m_max)
    irr.irr_set_tuning("mid_dmma", mid_dmma)
    shapes = [(151, 162), (151, 163), (153, 160), (160, 153), (96, 256), (256, 96), (97, 256),
              (77, 79), (78, 78), (79, 78), (110, 111), (111, 110), (64, 96), (95, 64),
              (1, 1024), (1024, 1), (33, 1), (1, 33), (300, 7), (7, 300), (1000, 30), (30, 1000)]
    _run_and_check(_uniform(shapes, seed=5))


@pytest.mark.parametrize("l1,nbo", [(1, 128), (0, 0), (0, 128)])
@pytest.mark.parametrize("nb", [5, 8, 16, 32, 64])
def test_tier_l_forced_small_nb(nb, l1, nbo):
    """Force everything through tier L (l1=1: CTA-per-matrix for m <= 256,
    l1=0: grid-wide kernel chain, one level (nbo 0) or two-level blocking):
    nb-1, nb, nb+1, 2nb+-1 sizes."""
    irr.irr_set_tuning("nb_outer", nbo)
    irr.irr_set_tuning("tier_s", 0)
    irr.irr_set_tuning("tier_m_max", 0)
    irr.irr_set_tuning("nb", nb)
    irr.irr_set_tuning("l1", l1)
    sizes = sorted({1, 2, nb - 1, nb, nb + 1, 2 * nb - 1, 2 * nb + 1, 3 * nb + 2} - {0})
    shapes = [(a, b) for a in sizes for b in sizes] + [(70, 45), (45, 70)]
    _run_and_check(_uniform(shapes, seed=nb))


def test_e1_replica_dcwi():
    """P:L167 Fig. 4: three matrices, the largest 15x15, nb = 5, three
    iterations; the second iteration sees full, partial and no work."""
    irr.irr_set_tuning("tier_s", 0)
    irr.irr_set_tuning("tier_m_max", 0)
    irr.irr_set_tuning("nb", 5)
    mats = _uniform([(15, 15), (8, 8), (4, 4)], seed=15)
    _run_and_check(mats)
    A, L, U, ipiv, _ = irrgen.g1_exact(1, 1, 15, 15)
    B, _, _, _, _ = irrgen.g1_exact(1, 2, 8, 8)
    Cm, _, _, _, _ = irrgen.g1_exact(1, 3, 4, 4)
    _run_and_check([A, B, Cm], exact=True)


def test_panel_in_global_memory():
    """Tall panels that do not fit shared memory take the in-place path."""
    irr.irr_set_tuning("panel_rows", 40)
    mats = _uniform([(300, 200), (200, 300), (257, 257), (100, 100)], seed=9)
    _run_and_check(mats)


@pytest.mark.parametrize("tier", ["default", "M", "Mdmma", "L", "L2", "L2two", "Ltall"])
def test_g1_exact_bitexact(tier):
    """G1: bit-exact L, U, ipiv in any arithmetic order."""
    if tier in ("M", "Mdmma"):
        irr.irr_set_tuning("tier_m_max", 24576)
        irr.irr_set_tuning("mid_dmma", 1 if tier == "Mdmma" else 0)
    if tier == "Ltall":
        irr.irr_set_tuning("l1_rows", 1024)
    if tier == "L2two":
        irr.irr_set_tuning("nb_outer", 128)
    if tier in ("L", "L2", "L2two", "Ltall"):
        irr.irr_set_tuning("tier_s", 0)
        irr.irr_set_tuning("tier_m_max", 0)
    if tier in ("L2", "L2two"):
        irr.irr_set_tuning("l1", 0)
    shapes = [(1, 1), (5, 5), (32, 32), (32, 17), (17, 32), (33, 33), (64, 20), (20, 64), (130, 130),
              (150, 160), (257, 100), (100, 257), (300, 300)]
    mats = [irrgen.g1_exact(3, g, m, n)[0] for g, (m, n) in enumerate(shapes)]
    _run_and_check(mats, exact=True)


def test_g1_singular_info():
    cases = [(6, 6, 0), (6, 6, 2), (32, 32, 31), (100, 100, 99), (64, 40, 17), (40, 64, 39), (300, 300, 150)]
    mats = [irrgen.g1_singular(4, g, m, n, c)[0] for g, (m, n, c) in enumerate(cases)]
    LUs, ipivs, info, _ = gpu_getrf(mats)
    for (m, n, c), A, LU, ip, inf in zip(cases, mats, LUs, ipivs, info):
        assert inf == c + 1
        check_getrf(A, LU, ip, int(inf), exact=True, label=f"sing {m}x{n}@{c}")


def test_g2_dominant_ipiv():
    shapes = [(1, 1), (5, 5), (32, 32), (64, 64), (300, 40), (40, 300), (256, 255), (200, 200), (500, 500)]
    for g, (m, n) in enumerate(shapes):
        A, ipiv = irrgen.g2_dominant(9, g, m, n)
        LUs, ipivs, info, _ = gpu_getrf([A])
        assert np.array_equal(ipivs[0], ipiv), (m, n)
        check_getrf(A, LUs[0], ipivs[0], int(info[0]), label=f"G2 {m}x{n}")


def test_g5_closed_forms():
    mats = [np.array([[3.5]]), np.array([[0.0]]), np.array([[0.5], [-3.0], [3.0], [1.0]]),
            np.array([[2.0, -1.0, 7.0]]), np.eye(9), np.eye(5)[[3, 0, 4, 1, 2]], np.zeros((4, 6)),
            np.zeros((40, 40)), np.eye(200)]
    _run_and_check(mats, exact=True)


@pytest.mark.parametrize("extra", [1, 7])
def test_leading_dimension(extra):
    shapes = [(5, 5), (31, 20), (64, 64), (100, 150), (300, 280)]
    _run_and_check(_uniform(shapes, seed=extra), ld_extra=extra)


def test_bad_arguments_are_skipped():
    """info < 0 for bad local dims; neighbours are unaffected."""
    mats = _uniform([(10, 10), (20, 20), (40, 30), (5, 5)], seed=3)
    m = [10, 20, 40, 5]
    n = [10, 20, 30, 5]
    m_bad = list(m)
    m_bad[1] = -3                       # bad m -> -1
    LUs, ipivs, info, _ = gpu_getrf(mats, m=m_bad, n=n, max_m=40, max_n=30)
    assert info[1] == -1
    for g in (0, 2, 3):
        check_getrf(mats[g], LUs[g], ipivs[g], int(info[g]))
    # larger than the required dims -> -1 / -2
    LUs, ipivs, info, _ = gpu_getrf(mats, max_m=30, max_n=30)
    assert info[2] == -1 and info[0] == 0


def test_required_dims_computed_on_device():
    mats = _uniform([(10, 12), (50, 40), (3, 3)], seed=8)
    LUs, ipivs, info, _ = gpu_getrf(mats, max_m=0, max_n=0)
    for A, LU, ip, inf in zip(mats, LUs, ipivs, info):
        check_getrf(A, LU, ip, int(inf))


def test_results_independent_of_batch_composition():
    """SURVEY §7 hard part 7 / G8: a matrix factors bitwise identically alone
    and inside a mixed batch (tier choice is a function of (m, n) only)."""
    shapes = [(20, 20), (100, 90), (300, 300), (7, 31)]
    mats = _uniform(shapes, seed=21)
    together, ip_t, _, _ = gpu_getrf(mats + _uniform([(256, 256)] * 3, seed=22))
    for g, A in enumerate(mats):
        alone, ip_a, _, _ = gpu_getrf([A])
        assert np.array_equal(alone[0], together[g]) and np.array_equal(ip_a[0], ip_t[g])


def test_c2_scaled_parity():
    """configs[1] shape (mixed square / rectangular, dims U{1..256}) on a 1/10 sample, every matrix."""
    cfg = irrgen.config("C2", scale=0.1)
    mats = [irrgen.uniform_values(cfg.seed, g, int(m), int(n)) for g, (m, n) in enumerate(zip(cfg.m, cfg.n))]
    st = _run_and_check(mats)
    assert st.get("match", 0) >= len(mats) - 3


@pytest.mark.parametrize("l1_rows", [256, 1024])
def test_c3_sample_parity(l1_rows):
    """configs[2] shape (square U{256..1024}), a sample of 12 matrices; with
    l1_rows = 1024 every one is factored by the CTA-per-matrix tier, whose
    panels above 256 rows run in place in global memory (panel_win)."""
    irr.irr_set_tuning("l1_rows", l1_rows)
    cfg = irrgen.config("C3", scale=0.006)
    mats = [irrgen.uniform_values(cfg.seed, g, int(m), int(n)) for g, (m, n) in enumerate(zip(cfg.m, cfg.n))]
    _run_and_check(mats)


@pytest.mark.parametrize("nb", [16, 32, 48, 64])
def test_windowed_panel_grid_tier(nb):
    """Grid-wide tier with the windowed register panel: every register
    variant (rows <= 512 / 1024 / 2048) and the > 2048 global fallback,
    tall, wide and square, window boundaries inside and at the panel edge."""
    irr.irr_set_tuning("l1", 0)
    irr.irr_set_tuning("nb", nb)
    irr.irr_set_tuning("nb_outer", 0)      # the one-level chain (two-level: test_two_level_grid_tier)
    shapes = [(700, 90), (1024, 64), (1025, 40), (1500, 33), (2048, 70), (2100, 40), (513, 513),
              (90, 700), (600, 600), (300, 17), (257, 257)]
    _run_and_check(_uniform(shapes, seed=31 + nb))


def test_windowed_panel_exact_and_singular():
    """G1 (bit-exact) and singular families through the windowed panel."""
    irr.irr_set_tuning("l1", 0)
    irr.irr_set_tuning("tier_s", 0)
    irr.irr_set_tuning("tier_m_max", 0)
    shapes = [(1100, 80), (2000, 64), (600, 600), (40, 1300)]
    mats = [irrgen.g1_exact(5, g, m, n)[0] for g, (m, n) in enumerate(shapes)]
    _run_and_check(mats, exact=True)
    cases = [(700, 700, 350), (1200, 90, 33), (520, 520, 0)]
    mats = [irrgen.g1_singular(6, g, m, n, c)[0] for g, (m, n, c) in enumerate(cases)]
    LUs, ipivs, info, _ = gpu_getrf(mats)
    for (m, n, c), A, LU, ip, inf in zip(cases, mats, LUs, ipivs, info):
        assert inf == c + 1
        check_getrf(A, LU, ip, int(inf), exact=True, label=f"sing {m}x{n}@{c}")


@pytest.mark.parametrize("win", [1, 0])
def test_grid_panel_variants_agree(win):
    """panel_win=1 (registers, global) and 0 (shared-memory / global getf2)."""
    irr.irr_set_tuning("l1", 0)
    irr.irr_set_tuning("panel_win", win)
    _run_and_check(_uniform([(800, 800), (300, 1000), (1000, 300)], seed=5))


def test_device_generator_matches_host():
    """irrgen.device (C5's on-device inputs) writes the same bytes as the host
    generator, for ld == m and ld > m, keyed by global id."""
    from irrgen import device as gdev
    rng = np.random.default_rng(3)
    m = rng.integers(0, 70, size=300)
    n = rng.integers(0, 70, size=300)
    ld = np.maximum(1, m) + rng.integers(0, 3, size=300) * (rng.random(300) < 0.3)
    gids = rng.permutation(10_000)[:300]
    off, total = irrgen.packed_offsets(ld, n)
    host = np.full(total, 7.0)
    irrgen.fill_packed(99, m, n, ld, off, host, gids=gids)
    dev = torch.full((total,), 7.0, dtype=torch.float64, device="cuda")
    gdev.Filler(99, m, n, ld, off, gids, dev.device).fill(dev)
    torch.cuda.synchronize()
    assert np.array_equal(dev.cpu().numpy().view(np.uint64), host.view(np.uint64))


@pytest.mark.parametrize("defer", [1, 0])
@pytest.mark.parametrize("l1", [1, 0])
def test_deferred_left_interchanges(defer, l1):
    """Left-block interchanges applied once at the end (default) and eagerly
    after every panel, in the CTA-per-matrix tier (l1=1) and the grid-wide
    tier (l1=0): both match the oracle and agree bitwise (interchanges only
    move values)."""
    irr.irr_set_tuning("l1", l1)
    irr.irr_set_tuning("nb_outer", 0)      # eager vs deferred exists on the one-level chain
    irr.irr_set_tuning("defer", defer)
    shapes = [(256, 256), (200, 240), (256, 70), (180, 256), (129, 200), (250, 33)]
    if not l1:
        shapes += [(700, 700), (1100, 300), (300, 900), (2000, 96)]
    mats = _uniform(shapes, seed=41)
    _run_and_check(mats)
    irr.irr_set_tuning("defer", 1 - defer)
    other, ip_o, _, _ = gpu_getrf(mats)
    irr.irr_set_tuning("defer", defer)
    mine, ip_m, _, _ = gpu_getrf(mats)
    for a, b, p, q in zip(mine, other, ip_m, ip_o):
        assert np.array_equal(a, b) and np.array_equal(p, q)


def test_c5_sample_parity():
    """configs[4] shapes (fronts 1..2048, heavy tail, full DGETRF): a
    stratified sample -- the largest fronts plus a random slice."""
    cfg = irrgen.config("C5")
    nf = cfg.m
    big = np.argsort(-nf)[:1]
    rest = np.random.default_rng(5).choice(len(nf), 40, replace=False)
    sel = np.unique(np.concatenate([big, rest]))
    mats = [irrgen.uniform_values(cfg.seed, int(g), int(cfg.m[g]), int(cfg.n[g])) for g in sel]
    st = _run_and_check(mats)
    assert st.get("match", 0) >= len(mats) - 2


def test_status_words():
    """a6 status words: info and the FNV-1a of ipiv (include/irr.h), checked
    against the host definition on the oracle's pivots; a bad-argument matrix
    gets (info, 0)."""
    from gpu_util import fnv1a_ipiv
    from paper_conf_sc_abdelfattahgbtld22_b200.batch import MatrixBatch
    import oracle
    shapes = [(5, 5), (40, 33), (300, 280), (1, 7), (0, 3)]
    mats = _uniform(shapes, seed=91)
    LUs, ipivs, info, (B, _) = gpu_getrf(mats)
    words = torch.zeros(2 * B.batch, dtype=torch.int32, device="cuda")
    irr.irr_status_words(B.batch, B.m, B.n, B.ipiv, B.info, words)
    w = words.cpu().numpy().view(np.uint32).reshape(-1, 2)
    for g, A in enumerate(mats):
        _, ipo, info_o, _ = oracle.getrf(A)
        assert int(w[g, 0]) == info_o
        assert int(w[g, 1]) == fnv1a_ipiv(ipo)
    # a matrix with a bad leading dimension: info -4, hash 0
    B.ld = torch.tensor([5, 40, 300, 0, 1], dtype=torch.int32, device="cuda")
    B.getrf()
    irr.irr_status_words(B.batch, B.m, B.n, B.ipiv, B.info, words)
    w = words.cpu().numpy().view(np.uint32).reshape(-1, 2)
    assert w[3, 0].view(np.int32) == -4 and w[3, 1] == 0


@pytest.mark.parametrize("chunks", [1, 3, 16])
def test_pipelined_host_entry_points(chunks):
    """getrf_host / getrf_partial_host (pinned host in -> host out, chunked
    H2D / getrf / D2H overlap) give bitwise the results of the device path."""
    from paper_conf_sc_abdelfattahgbtld22_b200.batch import (FrontBatch, MatrixBatch, getrf_host,
                                                             getrf_partial_host)
    cfg = irrgen.config("C2", scale=0.03)
    B = MatrixBatch(cfg.m, cfg.n)
    host = torch.zeros(B.total, dtype=torch.float64, pin_memory=True)
    irrgen.fill_packed(cfg.seed, cfg.m, cfg.n, B.ld_h, B.offsets, host.numpy())
    outs = [torch.empty(t.numel(), dtype=t.dtype, pin_memory=True) for t in (B.data, B.ipiv_data, B.info)]
    getrf_host(B, host, *outs, chunks=chunks)
    torch.cuda.synchronize()
    B.data.copy_(host)
    B.ipiv_data.zero_()
    B.getrf()
    torch.cuda.synchronize()
    assert np.array_equal(outs[0].numpy(), B.data.cpu().numpy())
    assert np.array_equal(outs[1].numpy(), B.ipiv_data.cpu().numpy())
    assert np.array_equal(outs[2].numpy(), B.info.cpu().numpy())
    n1, n2 = [3, 40, 0, 100, 7], [5, 60, 9, 30, 0]
    F = FrontBatch(n1, n2)
    fh = torch.zeros(F.total, dtype=torch.float64, pin_memory=True)
    irrgen.fill_packed(7, F.nf_h, F.nf_h, F.ld_h, F.offsets, fh.numpy())
    fo = [torch.empty(t.numel(), dtype=t.dtype, pin_memory=True) for t in (F.data, F.ipiv_data, F.info)]
    getrf_partial_host(F, fh, *fo, chunks=chunks)
    torch.cuda.synchronize()
    F.data.copy_(fh)
    F.getrf_partial()
    torch.cuda.synchronize()
    assert np.array_equal(fo[0].numpy(), F.data.cpu().numpy())
    assert np.array_equal(fo[2].numpy(), F.info.cpu().numpy())


@pytest.mark.parametrize("split", [0, 1])
@pytest.mark.parametrize("nb,nbo", [(32, 128), (32, 64), (16, 64), (32, 96), (16, 128)])
def test_two_level_grid_tier(nb, nbo, split):
    """Grid-wide tier with two-level blocking: inner panels of nb confined to
    outer blocks of nbo, then one interchange + U12 solve + K = nbo GEMM
    update of the rest per outer block.  Ragged outer / inner tails, tall,
    wide, K < nbo, widths that end inside an outer block."""
    irr.irr_set_tuning("l1", 0)
    irr.irr_set_tuning("nb", nb)
    irr.irr_set_tuning("nb_outer", nbo)
    irr.irr_set_tuning("split_strip", split)  # 1: inner trailing update as a grid-wide GEMM
    shapes = [(700, 90), (1024, 64), (1025, 40), (1500, 33), (2048, 70), (513, 513), (90, 700), (600, 600),
              (300, 17), (257, 257), (1000, 1000), (129, 400), (400, 129), (2000, 1300), (nbo + 1, nbo + 1),
              (3 * nbo - 1, 3 * nbo + 5)]
    _run_and_check(_uniform(shapes, seed=77 + nb + nbo))


def test_two_level_exact_and_singular():
    """G1 bit-exact and exact-singular through the two-level grid tier."""
    irr.irr_set_tuning("l1", 0)
    irr.irr_set_tuning("tier_s", 0)
    irr.irr_set_tuning("tier_m_max", 0)
    irr.irr_set_tuning("nb_outer", 128)
    shapes = [(1100, 300), (2000, 260), (600, 600), (140, 1300), (1024, 1024)]
    mats = [irrgen.g1_exact(15, g, m, n)[0] for g, (m, n) in enumerate(shapes)]
    _run_and_check(mats, exact=True)
    cases = [(700, 700, 350), (1200, 300, 129), (520, 520, 0), (900, 900, 127)]
    mats = [irrgen.g1_singular(16, g, m, n, c)[0] for g, (m, n, c) in enumerate(cases)]
    LUs, ipivs, info, _ = gpu_getrf(mats)
    for (m, n, c), A, LU, ip, inf in zip(cases, mats, LUs, ipivs, info):
        assert inf == c + 1
        check_getrf(A, LU, ip, int(inf), exact=True, label=f"sing {m}x{n}@{c}")


def test_results_bitwise_identical_across_shard_counts():
    """a C5-shaped batch factored as G = 1, 2, 4, 8 LPT
    shards (one irr_getrf per shard, inputs keyed by global id) gives
    bitwise the same factors, pivots and status words per global matrix."""
    from paper_conf_sc_abdelfattahgbtld22_b200 import flops as F
    from paper_conf_sc_abdelfattahgbtld22_b200.batch import MatrixBatch
    from paper_conf_sc_abdelfattahgbtld22_b200.shard import lpt_partition
    cfg = irrgen.config("C5", scale=0.01)
    w = F.getrf_flops(cfg.m, cfg.n)
    ref = None
    for G in (1, 2, 4, 8):
        owner = lpt_partition(w, G)
        got = {}
        for r in range(G):
            mine = np.nonzero(owner == r)[0]
            B = MatrixBatch(cfg.m[mine], cfg.n[mine])
            host = np.zeros(B.total)
            irrgen.fill_packed(cfg.seed, cfg.m[mine], cfg.n[mine], B.ld_h, B.offsets, host, gids=mine)
            B.data.copy_(torch.from_numpy(host))
            B.getrf()
            words = torch.zeros(2 * B.batch, dtype=torch.int32, device="cuda")
            irr.irr_status_words(B.batch, B.m, B.n, B.ipiv, B.info, words)
            torch.cuda.synchronize()
            out, ip = B.data.cpu().numpy(), B.ipiv_data.cpu().numpy()
            wd = words.cpu().numpy().reshape(-1, 2)
            for q, g in enumerate(mine):
                got[int(g)] = (np.array(B.matrix(q, out)).tobytes(), np.array(B.ipiv_of(q, ip)).tobytes(),
                               tuple(wd[q]))
        if ref is None:
            ref = got
        else:
            assert got == ref, f"G = {G} differs from G = 1"


@pytest.mark.parametrize("part_grid", [1, 2])
def test_two_parts_bitwise_equal(part_grid):
    """The two-level grid tier split into two LPT halves on two streams
    (tuning parts = 2) factors every matrix bitwise as the single list does
    (the per-matrix arithmetic does not depend on the part), and matches the
    oracle."""
    shapes = [(700, 700), (300, 260), (1024, 900), (520, 520), (2000, 300), (300, 2000), (45, 45), (600, 601),
              (1500, 1500)]
    mats = _uniform(shapes, seed=97)
    one, ip1, inf1, _ = gpu_getrf(mats)
    irr.irr_set_tuning("parts", 2)
    irr.irr_set_tuning("part_grid", part_grid)
    two, ip2, inf2, _ = gpu_getrf(mats)
    for a, b, p, q in zip(one, two, ip1, ip2):
        assert np.array_equal(a, b) and np.array_equal(p, q)
    assert np.array_equal(inf1, inf2)
    _run_and_check(mats)


@pytest.mark.parametrize("cols", [32, 64])
def test_outer_strip_widths(cols):
    """The two-level interchange + U12 solve in 32-column strips (packed L11,
    2 CTAs / SM) and 64-column strips (square L11, 1 CTA / SM): oracle parity
    and G1 bit-exactness."""
    irr.irr_set_tuning("l1", 0)
    irr.irr_set_tuning("outer_cols", cols)
    shapes = [(700, 700), (300, 1000), (1000, 300), (513, 513), (1300, 1300), (129, 900)]
    _run_and_check(_uniform(shapes, seed=101 + cols))
    mats = [irrgen.g1_exact(17, g, m, n)[0] for g, (m, n) in enumerate([(600, 600), (300, 700), (900, 400)])]
    _run_and_check(mats, exact=True)


def test_outer_update_vs_oracle():
    """The two-level outer update against the oracle on shapes with ragged
    outer tails, wide / tall, several strips and row tiles, pivots from below
    and from the block."""
    irr.irr_set_tuning("l1", 0)
    shapes = [(700, 700), (300, 1000), (1000, 300), (513, 513), (1300, 1300), (129, 900), (2048, 2048),
              (1500, 1100), (260, 2000), (640, 129), (2000, 640)]
    _run_and_check(_uniform(shapes, seed=303))


@pytest.mark.parametrize("seed", [1, 2])
def test_grouped_tier_s_bitwise_and_oracle(seed):
    """tier_s = 2 packs 4 (m, n <= 8) or 2 (m, n <= 16) matrices per warp.
    Each row sees the same FMA sequence as the warp-per-matrix kernel
    (tier_s = 1): results bitwise identical, and every matrix matches the
    oracle.  Mixed shapes so a warp's matrices differ in K and n (groups that
    sit steps out), rectangular both ways, tall n <= 8 with m > 16 (stays on
    the warp-per-matrix kernels), and a batch that is not a multiple of the
    group count."""
    rng = np.random.default_rng(seed)
    shapes = [(int(rng.integers(1, 9)), int(rng.integers(1, 9))) for _ in range(203)]
    shapes += [(int(rng.integers(1, 17)), int(rng.integers(1, 17))) for _ in range(151)]
    shapes += [(int(rng.integers(17, 33)), int(rng.integers(1, 9))) for _ in range(23)]
    shapes += [(int(rng.integers(1, 33)), int(rng.integers(17, 33))) for _ in range(97)]
    shapes += [(int(rng.integers(17, 33)), int(rng.integers(1, 33))) for _ in range(61)]
    shapes += [(m, n) for m in (1, 2, 7, 8, 9, 15, 16) for n in (1, 2, 7, 8, 9, 15, 16)]
    mats = _uniform(shapes, seed=100 + seed)
    sing = [irrgen.g1_singular(5, g, 8, 8, c)[0] for g, c in enumerate((0, 3, 7))]
    sing += [irrgen.g1_singular(6, g, 16, 16, c)[0] for g, c in enumerate((1, 12, 15))]
    sing += [irrgen.g1_singular(7, g, 32, 32, c)[0] for g, c in enumerate((0, 16, 31))]
    sing += [irrgen.g1_exact(8, g, m, n)[0] for g, (m, n) in enumerate(((32, 32), (17, 32), (32, 17), (31, 25)))]
    mats += sing
    irr.irr_set_tuning("tier_s", 1)
    LU1, ip1, info1, _ = gpu_getrf(mats)
    for ts in (2,):
        irr.irr_set_tuning("tier_s", ts)
        LU2, ip2, info2, _ = gpu_getrf(mats)
        assert np.array_equal(info1, info2), ts
        for a, b, p, q in zip(LU1, LU2, ip1, ip2):
            assert np.array_equal(p, q), ts
            assert np.array_equal(a.view(np.int64), b.view(np.int64)), ts
    for g, (A, LU, ip, inf) in enumerate(zip(mats, LU2, ip2, info2)):
        check_getrf(A, LU, ip, int(inf), exact=g >= len(mats) - len(sing), label=f"grouped #{g} {A.shape}")


@pytest.mark.parametrize("warps", [8, 16, "tma"])
def test_xgemm_variants_bitwise_equal(warps):
    """The two-level trailing GEMM on the 8-warp or the 16-warp core gives
    bitwise the factors of the default warp-specialised core (9: 8 DMMA warps
    + a producer warpgroup on an mbarrier ring; same DMMA sequence per
    accumulator), and matches the oracle; "tma": the default core with the A
    operand staged by cp.async.bulk (odd and even leading dimensions, ragged
    row tiles, K tails)."""
    irr.irr_set_tuning("l1", 0)
    shapes = [(700, 700), (300, 1000), (1000, 300), (1300, 1300), (2048, 2048), (129, 900), (2000, 640),
              (1001, 1001), (777, 901), (1290, 1290), (513, 700)]
    mats = _uniform(shapes, seed=404)
    one, ip1, inf1, _ = gpu_getrf(mats)
    if warps == "tma":  # the warp-specialised core with the A operand by TMA bulk copies
        irr.irr_set_tuning("xgemm_tma", 1)
    else:
        irr.irr_set_tuning("xgemm_warps", warps)
    two, ip2, inf2, _ = gpu_getrf(mats)
    for a, b, p, q in zip(one, two, ip1, ip2):
        assert np.array_equal(a.view(np.int64), b.view(np.int64)) and np.array_equal(p, q)
    assert np.array_equal(inf1, inf2)
    _run_and_check(mats)

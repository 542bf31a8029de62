"""GPU parity of irr_extend_add (§III-A: the child's Schur complement
is scattered into the parent front; L102: one tree level at once) through the
C ABI against oracle.extend_add applied child by child.

Bar: bit-exact.  One FP64 add per parent entry per call (sibling rounds) is
exactly fl(Fp + F22) whatever the schedule; with several children of one
parent in one call the adds are atomic in an unspecified order, so that case
is checked bit-exact on integer-valued data (every partial sum exact) and
within 2 * eps * (|Fp| + sum |contributions|) on dyadic data.
"""
import numpy as np
import pytest

import irrgen
import oracle

pytestmark = pytest.mark.gpu

torch = pytest.importorskip("torch")
if not torch.cuda.is_available():
    pytest.skip("no CUDA device", allow_module_level=True)

from paper_conf_sc_abdelfattahgbtld22_b200 import irr  # noqa: E402
from ea_util import Level  # noqa: E402

EPS = np.finfo(np.float64).eps


def _run(L, sel, max_n2=None):
    a = L.args(sel)
    mx = int(max(L.n2[list(sel)])) if max_n2 is None else max_n2
    irr.irr_extend_add(a["batch"], mx, a["n2"], a["F22"], a["ld22"], a["rel"], a["np_"], a["Fp"], a["ldp"],
                       a["info"])
    torch.cuda.synchronize()
    return a["info"].cpu().numpy()[: a["batch"]]


def _oracle(lvl, order):
    nps, parent, n2, rel, F22, Fp = lvl
    out = [F.copy(order="F") for F in Fp]
    for c in order:
        out[parent[c]] = oracle.extend_add(out[parent[c]], F22[c], rel[c])
    return out


@pytest.mark.parametrize("np_max", [300, 85])
@pytest.mark.parametrize("ld_extra", [0, 3])
def test_sibling_rounds_bit_exact(ld_extra, np_max):
    """Round r = the r-th child of every parent: one add per entry per call.
    np_max 85 keeps every child <= 64 (the warp-per-child kernel, both rel
    registers in use); 300 takes the CTA-per-child kernel."""
    lvl = irrgen.extend_add_level(11, 40, np_max)
    nps, parent, n2, rel, F22, Fp = lvl
    L = Level(*lvl, ld_extra=ld_extra)
    kids = np.arange(len(parent))
    r0, r1 = kids[0::2], kids[1::2]
    assert np.all(_run(L, r0) == 0) and np.all(_run(L, r1) == 0)
    want = _oracle(lvl, list(r0) + list(r1))
    got = L.parents_host()
    for p in range(len(nps)):
        assert np.array_equal(got[p], want[p]), p


def test_shared_parents_one_call():
    nps, parent, n2, rel, F22, Fp = irrgen.extend_add_level(12, 30, 260, children_per_parent=3)
    # integer-valued: any summation order is exact
    F22i = [np.round(F * 1024) for F in F22]
    Fpi = [np.round(F * 1024) for F in Fp]
    lvl = (nps, parent, n2, rel, F22i, Fpi)
    L = Level(*lvl)
    assert np.all(_run(L, range(len(parent))) == 0)
    want = _oracle(lvl, range(len(parent)))
    got = L.parents_host()
    for p in range(len(nps)):
        assert np.array_equal(got[p], want[p]), p
    # dyadic values: within the rounding of a 4-term sum in any order
    lvl = (nps, parent, n2, rel, F22, Fp)
    L = Level(*lvl)
    _run(L, range(len(parent)))
    want = _oracle(lvl, range(len(parent)))
    bound = [np.abs(F).copy(order="F") for F in Fp]
    for c in range(len(parent)):
        bound[parent[c]] = oracle.extend_add(bound[parent[c]], np.abs(F22[c]), rel[c])
    got = L.parents_host()
    for p in range(len(nps)):
        assert np.all(np.abs(got[p] - want[p]) <= 4 * EPS * bound[p]), p


def test_large_child_beyond_shared_rel():
    """n2 > 4096: rel entries past the shared-memory stage come from global."""
    rng = np.random.default_rng(4)
    npp, n2 = 4700, 4500
    rel = np.sort(rng.choice(npp, size=n2, replace=False)).astype(np.int32)
    Fp = irrgen.uniform_values(4, 1, npp, npp)
    F22 = irrgen.uniform_values(4, 2, n2, n2)
    lvl = (np.array([npp]), np.array([0]), np.array([n2]), [rel], [F22], [Fp])
    L = Level(*lvl)
    assert np.all(_run(L, [0]) == 0)
    assert np.array_equal(L.parents_host()[0], oracle.extend_add(Fp, F22, rel))


def test_tiny_children_and_edge_cases():
    """n2 = 1 / 2 / 0 children, np = 1 parents, a bad map (-6), n2 > max_n2 (-3)."""
    nps = np.array([1, 5, 9, 9])
    Fp = [irrgen.uniform_values(7, 10 + p, int(s), int(s)) for p, s in enumerate(nps)]
    parent = np.array([0, 1, 2, 3, 2, 1])
    n2 = np.array([1, 2, 0, 3, 4, 1])
    rel = [np.array([0]), np.array([1, 4]), np.array([], np.int32), np.array([0, 9, 2]), np.array([1, 2, 5, 8]),
           np.array([3])]
    F22 = [irrgen.uniform_values(7, c, int(k), int(k)) for c, k in enumerate(n2)]
    L = Level(nps, parent, n2, rel, F22, Fp)
    info = _run(L, range(6), max_n2=4)
    assert list(info) == [0, 0, 0, -6, 0, 0]
    good = [0, 1, 2, 4, 5]
    want = _oracle((nps, parent, n2, rel, F22, Fp), good)
    got = L.parents_host()
    for p in range(4):
        assert np.array_equal(got[p], want[p]), p
    info = _run(L, [4], max_n2=3)
    assert list(info) == [-3]
    assert np.array_equal(L.parents_host()[2], got[2])


def test_host_argument_errors():
    z = torch.zeros(4, dtype=torch.int32, device="cuda")
    assert irr.irr_extend_add(-1, 1, z, z, z, z, z, z, z, z, check=False) == -1
    assert irr.irr_extend_add(1, -1, z, z, z, z, z, z, z, z, check=False) == -2
    assert irr.irr_extend_add(1, 1, z, None, z, z, z, z, z, z, check=False) == -4
    assert irr.irr_extend_add(0, 0, None, None, None, None, None, None, None, None, check=False) == 0

"""The level-by-level assembly-tree traversal (PAPER.md
L93-102 §III-A: partial factorization of every front of a level, then the
extend-add of the Schur complements into the parents, leaves to root),
through the C ABI (tree.AssemblyTree: irr_getrf_partial + irr_extend_add per
level), against the oracle chained the same way (oracle.getrf_partial per
front, oracle.extend_add per child in the same sibling order)."""
import numpy as np
import pytest

import irrgen
import oracle

pytestmark = pytest.mark.gpu

torch = pytest.importorskip("torch")
if not torch.cuda.is_available():
    pytest.skip("no CUDA device", allow_module_level=True)

from gpu_util import check_partial, rel_dev  # noqa: E402
from paper_conf_sc_abdelfattahgbtld22_b200 import irr  # noqa: E402
from paper_conf_sc_abdelfattahgbtld22_b200.tree import AssemblyTree  # noqa: E402


@pytest.fixture(autouse=True)
def _reset_tuning():
    irr.irr_reset_tuning()
    yield
    irr.irr_reset_tuning()


def _load(T, fronts):
    host = np.zeros(T.F.total)
    for v, Fv in enumerate(fronts):
        if Fv.size:
            T.F.front(T.pos[v], host)[:, :] = Fv
    T.F.data.copy_(torch.from_numpy(host))


def _fronts(T, n):
    out = T.F.data.cpu().numpy()
    return [np.array(T.F.front(T.pos[v], out)) for v in range(n)]


def _ipiv(T, v):
    return np.array(T.F.ipiv_of(T.pos[v], T.F.ipiv_data.cpu().numpy()))


def _sibling_order(tree, level):
    """Children of `level` in the driver's round order (round r = r-th child of each parent)."""
    seen, rounds = {}, []
    for v in tree.levels[level]:
        p = int(tree.parent[v])
        if p < 0:
            continue
        r = seen.get(p, 0)
        seen[p] = r + 1
        while len(rounds) <= r:
            rounds.append([])
        rounds[r].append(int(v))
    return [v for rnd in rounds for v in rnd]


@pytest.mark.parametrize("depth", [3, 6])
def test_tree_exact(depth):
    """Exact dyadic tree: every assembled front is a G1' front, so after the
    traversal every node holds exactly its chosen factors: F11 -> L\\U with the
    chosen ipiv, F12 -> X, F22 -> S, F21 = the assembled F21."""
    tree = irrgen.assembly_tree(40 + depth, depth, s0=6.0)
    orig, exp = irrgen.tree_exact(41, tree)
    T = AssemblyTree(tree.n1, tree.n2, tree.parent, tree.rel, tree.levels)
    _load(T, orig)
    T.factor()
    torch.cuda.synchronize()
    assert all((i.cpu().numpy() == 0).all() for i in T.extend_add_info())
    assert (T.F.info.cpu().numpy()[: T.F.batch] == 0).all()
    got = _fronts(T, len(orig))
    for v, (G, e) in enumerate(zip(got, exp)):
        a = int(tree.n1[v])
        LU = np.tril(e["L"], -1) + e["U"]
        assert np.array_equal(G[:a, :a], LU), f"node {v}: F11"
        assert np.array_equal(G[:a, a:], e["X"]), f"node {v}: F12"
        assert np.array_equal(G[a:, a:], e["S"]), f"node {v}: F22"
        assert np.array_equal(G[a:, :a], e["F21"]), f"node {v}: F21"
        assert np.array_equal(_ipiv(T, v), e["ipiv"]), f"node {v}: ipiv"


def test_tree_uniform_vs_oracle_chain():
    """Uniform fronts, depth 7: level by level, (1) the GPU's assembled fronts
    match the oracle chain's (1e-10 relative to the front's scale), (2) every
    front's partial factorization matches the oracle on the GPU's own
    assembled input (north_star tolerances, Q12), (3) the root matches the
    oracle chain end to end (1e-10 relative, L and U of the root's F11)."""
    tree = irrgen.assembly_tree(7, 7, s0=10.0)
    vals = irrgen.tree_values(8, tree)
    T = AssemblyTree(tree.n1, tree.n2, tree.parent, tree.rel, tree.levels)
    _load(T, vals)
    ora = [F.copy(order="F") for F in vals]
    n = len(vals)
    for level, lv in enumerate(tree.levels):
        torch.cuda.synchronize()
        assembled = _fronts(T, n)
        for v in lv:
            scale = max(1e-300, np.abs(ora[v]).max())
            d = np.abs(assembled[v] - ora[v]).max() / scale
            assert d <= 1e-10, f"level {level} node {v}: assembled front deviates {d}"
        T.partial(level)
        torch.cuda.synchronize()
        after = _fronts(T, n)
        info = T.F.info.cpu().numpy()
        for v in lv:
            a = int(tree.n1[v])
            check_partial(assembled[v], a, after[v], _ipiv(T, v), int(info[T.pos[v]]), label=f"L{level} node {v}")
            # the oracle chain: same step on its own assembled front
            o = ora[v]
            o11, o12, o22, _, _ = oracle.getrf_partial(o[:a, :a], o[:a, a:], o[a:, :a], o[a:, a:])
            o[:a, :a], o[:a, a:], o[a:, a:] = o11, o12, o22
        T.extend_add(level)
        for c in _sibling_order(tree, level):
            p, a = int(tree.parent[c]), int(tree.n1[c])
            ora[p] = oracle.extend_add(ora[p], ora[c][a:, a:], tree.rel[c])
    torch.cuda.synchronize()
    assert all((i.cpu().numpy() == 0).all() for i in T.extend_add_info())
    root = int(tree.levels[-1][0])
    G = _fronts(T, n)[root]
    assert rel_dev(np.tril(G, -1), np.tril(ora[root], -1)) <= 1e-10
    assert rel_dev(np.triu(G), np.triu(ora[root])) <= 1e-10

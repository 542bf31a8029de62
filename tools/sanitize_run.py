"""One small call of a library entry point, for compute-sanitizer
(memcheck / racecheck / synccheck) runs: every tier and building block on a
tiny seeded batch, results checked against the oracle so a sanitizer run also
confirms the outputs.

    python tools/sanitize_run.py <what>
    what: tierS tierM L1 grid1 grid2 partial partial_lapack getrs getrs_vec extend_add zgetrf tree
"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
sys.path.insert(0, os.path.join(os.path.dirname(os.path.dirname(os.path.abspath(__file__))), "tests"))
import numpy as np  # noqa: E402
import torch  # noqa: E402

import irrgen  # noqa: E402
import oracle  # noqa: E402
from paper_conf_sc_abdelfattahgbtld22_b200 import irr  # noqa: E402

what = sys.argv[1]
# extra tuning for the run: IRR_TUNE="key=value,key=value"
for kv in filter(None, os.environ.get("IRR_TUNE", "").split(",")):
    k, v = kv.split("=")
    irr.irr_set_tuning(k, int(v))


def getrf_check(shapes, **tune):
    from gpu_util import check_getrf, gpu_getrf
    for k, v in tune.items():
        irr.irr_set_tuning(k, v)
    mats = [irrgen.uniform_values(7, g, m, n) for g, (m, n) in enumerate(shapes)]
    LUs, ipivs, info, _ = gpu_getrf(mats)
    for A, LU, ip, inf in zip(mats, LUs, ipivs, info):
        check_getrf(A, LU, ip, int(inf))


rng = np.random.default_rng(1)
if what == "tierS":
    getrf_check([(int(a), int(a)) for a in rng.integers(1, 33, 40)] + [(32, 17), (17, 32), (5, 9)])
elif what == "tierM":
    getrf_check([(int(a), int(b)) for a, b in zip(rng.integers(33, 80, 20), rng.integers(33, 80, 20))])
elif what == "L1":
    getrf_check([(int(a), int(b)) for a, b in zip(rng.integers(120, 257, 8), rng.integers(120, 300, 8))])
elif what == "grid1":
    getrf_check([(300, 300), (520, 400), (400, 520), (700, 90)], l1=0, nb_outer=0)
elif what == "grid2":
    getrf_check([(300, 300), (520, 400), (400, 520), (700, 90), (90, 700), (401, 333)], l1=0, nb_outer=128)
elif what in ("partial", "partial_lapack"):
    from gpu_util import check_partial, gpu_partial
    shapes = [(3, 4), (17, 40), (50, 80), (129, 200), (300, 150)]
    fronts = [(irrgen.front_values(8, g, a + b), a) for g, (a, b) in enumerate(shapes)]
    out, ipivs, info = gpu_partial(fronts, lapack=(what == "partial_lapack"))
    if what == "partial":
        for (F, a), Fg, ip, inf in zip(fronts, out, ipivs, info):
            check_partial(F, a, Fg, ip, int(inf))
elif what in ("getrs", "getrs_vec"):
    from paper_conf_sc_abdelfattahgbtld22_b200.batch import MatrixBatch
    ns = [1, 31, 64, 100, 257]
    r = 1 if what == "getrs_vec" else 7
    FA, RB = MatrixBatch(ns, ns), MatrixBatch(ns, [r] * len(ns))
    for B, seed, cols in ((FA, 3, ns), (RB, 4, [r] * len(ns))):
        host = np.zeros(B.total)
        for i, (n, c) in enumerate(zip(ns, cols)):
            B.matrix(i, host)[:, :] = irrgen.uniform_values(seed, i, n, c)
        B.data.copy_(torch.from_numpy(host))
    FA.getrf()
    st = FA.getrs(RB)
    torch.cuda.synchronize()
    assert (st.cpu().numpy()[: FA.batch] == 0).all()
elif what == "extend_add":
    from ea_util import Level
    lvl = irrgen.extend_add_level(11, 12, 200)
    L = Level(*lvl)
    kids = np.arange(len(lvl[1]))
    for sel in (kids[0::2], kids[1::2]):
        a = L.args(sel)
        irr.irr_extend_add(a["batch"], int(max(L.n2[list(sel)])), a["n2"], a["F22"], a["ld22"], a["rel"], a["np_"],
                           a["Fp"], a["ldp"], a["info"])
    torch.cuda.synchronize()
elif what == "zgetrf":
    from paper_conf_sc_abdelfattahgbtld22_b200.batch import ZMatrixBatch
    shapes = [(7, 7), (40, 33), (64, 64), (100, 130)]
    B = ZMatrixBatch([s[0] for s in shapes], [s[1] for s in shapes])
    host = np.zeros(B.total)
    mats = [irrgen.zuniform_values(5, g, m, n) for g, (m, n) in enumerate(shapes)]
    for i, A in enumerate(mats):
        B.matrix(i, host)[:, :] = A
    B.data.copy_(torch.from_numpy(host))
    B.getrf()
    torch.cuda.synchronize()
    ip = B.ipiv_data.cpu().numpy()
    for i, A in enumerate(mats):
        assert np.array_equal(np.array(B.ipiv_of(i, ip)), oracle.zgetrf(A)[1])
elif what == "tree":
    from paper_conf_sc_abdelfattahgbtld22_b200.tree import AssemblyTree
    tree = irrgen.assembly_tree(3, 4, s0=6.0)
    T = AssemblyTree(tree.n1, tree.n2, tree.parent, tree.rel, tree.levels)
    T.F.data.copy_(torch.rand(T.F.total, dtype=torch.float64, device="cuda") * 2 - 1)
    T.factor()
    torch.cuda.synchronize()
else:
    raise SystemExit(f"unknown {what}")
print("ok", what)

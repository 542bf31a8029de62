"""Device marshalling for the extend-add tests and tools/bench_extend_add.py:
column-major matrices as (n, ld) row-major torch tensors, pointer arrays."""
import numpy as np
import torch


def to_dev(M, ld_extra=0):
    m, n = M.shape
    ld = max(1, m + ld_extra)
    T = torch.full((max(n, 1), ld), float("nan"), dtype=torch.float64, device="cuda")
    if M.size:
        T[:n, :m] = torch.from_numpy(np.ascontiguousarray(M.T))
    return T, ld


def from_dev(T, m, n):
    return T.cpu().numpy()[:n, :m].T.copy(order="F")


def ptrs(ts):
    return torch.tensor([t.data_ptr() for t in ts], dtype=torch.int64, device="cuda")


def i32(x):
    return torch.tensor(np.asarray(x, dtype=np.int32), dtype=torch.int32, device="cuda")


class Level:
    """Parents and children of one tree level resident on the device."""

    def __init__(self, np_sizes, parent, n2, rel, F22, Fp, ld_extra=0):
        self.np_sizes = np.asarray(np_sizes)
        self.Pt, ldp = zip(*[to_dev(F, ld_extra) for F in Fp]) if len(Fp) else ((), ())
        self.ldp_of = list(ldp)
        self.Ct, ld22 = zip(*[to_dev(F, ld_extra) for F in F22]) if len(F22) else ((), ())
        self.rel_t = [torch.tensor(np.asarray(r, dtype=np.int32), dtype=torch.int32, device="cuda")
                      if len(r) else torch.zeros(1, dtype=torch.int32, device="cuda") for r in rel]
        self.parent, self.n2, self.ld22 = np.asarray(parent), np.asarray(n2), list(ld22)

    def args(self, sel):
        sel = list(sel)
        p = [int(self.parent[c]) for c in sel]
        return dict(
            batch=len(sel),
            n2=i32([self.n2[c] for c in sel]),
            F22=ptrs([self.Ct[c] for c in sel]),
            ld22=i32([self.ld22[c] for c in sel]),
            rel=ptrs([self.rel_t[c] for c in sel]),
            np_=i32([self.np_sizes[q] for q in p]),
            Fp=ptrs([self.Pt[q] for q in p]),
            ldp=i32([self.ldp_of[q] for q in p]),
            info=torch.full((max(1, len(sel)),), 99, dtype=torch.int32, device="cuda"),
        )

    def parents_host(self):
        return [from_dev(T, int(s), int(s)) for T, s in zip(self.Pt, self.np_sizes)]

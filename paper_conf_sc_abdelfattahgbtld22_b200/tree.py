"""Level-by-level traversal of an assembly tree on the GPU (SURVEY §8(f)
NEXT 2; §III-A).

"STRUMPACK traverses the tree level-by-level, from leaves to root" (L102):
every front of one level is partially factored by ONE irr_getrf_partial call
(F11 -> L\\U, F12 <- U^-1 L^-1 P^T F12, F22 <- F22 - F21 F12, L95-97), then
the Schur complements F22 of that level are scattered into their parents by
irr_extend_add (L99), one call per sibling round so that every parent entry
receives at most one contribution per call (bit-identical to the sequential
order, include/irr.h).  The host only walks the levels; every step of the
path runs in the library's kernels through the C ABI.

Layout (caller-side setup, like batch.FrontBatch): all fronts of all levels
in one FrontBatch, level by level; the child -> parent pointer / size arrays
of every sibling round built once on the device.
"""
from __future__ import annotations

import numpy as np
import torch

from . import irr
from .batch import FrontBatch


class AssemblyTree:
    def __init__(self, n1, n2, parent, rel, levels, device="cuda"):
        self.levels = [np.asarray(l, dtype=np.int64) for l in levels]
        order = np.concatenate(self.levels)
        self.node_order = order
        pos = np.empty(len(order), dtype=np.int64)
        pos[order] = np.arange(len(order))
        self.pos = pos                      # node -> slot in the FrontBatch
        n1 = np.asarray(n1, dtype=np.int64)
        n2 = np.asarray(n2, dtype=np.int64)
        parent = np.asarray(parent, dtype=np.int64)
        self.F = F = FrontBatch(n1[order], n2[order], device=device)
        dev = F.device
        bounds = np.cumsum([0] + [len(l) for l in self.levels])
        self.slices = [(int(a), int(b)) for a, b in zip(bounds[:-1], bounds[1:])]
        # index maps, one flat int32 device buffer
        roff = np.zeros(len(order) + 1, dtype=np.int64)
        roff[1:] = np.cumsum([max(1, len(rel[v])) for v in order])
        flat = np.zeros(int(roff[-1]), dtype=np.int32)
        for q, v in enumerate(order):
            if len(rel[v]):
                flat[roff[q]: roff[q] + len(rel[v])] = rel[v]
        self.rel_data = torch.from_numpy(flat).to(dev)
        rel_ptr = self.rel_data.data_ptr() + 4 * roff[:-1]
        base = F.data.data_ptr() + 8 * F.offsets          # front q's F11 = the whole block
        # per level: sibling rounds of the children whose parent is a front
        self.rounds = []
        for lv in self.levels:
            kids = [int(v) for v in lv if parent[v] >= 0]
            rounds = []
            seen = {}
            for v in kids:
                r = seen.get(int(parent[v]), 0)
                seen[int(parent[v])] = r + 1
                while len(rounds) <= r:
                    rounds.append([])
                rounds[r].append(v)
            lvl = []
            for rnd in rounds:
                q = pos[np.asarray(rnd)]
                p = pos[parent[np.asarray(rnd)]]

                def T(x, dt):
                    return torch.from_numpy(np.ascontiguousarray(x, dtype=dt)).to(dev)
                lvl.append(dict(
                    batch=len(rnd), max_n2=int(F.n2_h[q].max()),
                    n2=T(F.n2_h[q], np.int32), F22=F.F22[torch.from_numpy(q).to(dev)],
                    ld22=T(F.ld_h[q], np.int32), rel=T(rel_ptr[q], np.int64),
                    np_=T(F.nf_h[p], np.int32), Fp=T(base[p], np.int64), ldp=T(F.ld_h[p], np.int32),
                    info=torch.zeros(max(1, len(rnd)), dtype=torch.int32, device=dev)))
            self.rounds.append(lvl)

    # -- the two steps of one level (exposed for the level-by-level tests)
    def partial(self, level: int, stream=None):
        """irr_getrf_partial on every front of `level` (one call)."""
        F = self.F
        a, b = self.slices[level]
        if b <= a:
            return
        S = lambda t: t[a:b]  # noqa: E731
        irr.irr_getrf_partial(b - a, int(F.n1_h[a:b].max()), int(F.n2_h[a:b].max()), S(F.n1), S(F.n2),
                              S(F.F11), S(F.ld11), S(F.F12), S(F.ld12), S(F.F21), S(F.ld21), S(F.F22),
                              S(F.ld22), S(F.ipiv), S(F.info), F.workspace(), stream)

    def extend_add(self, level: int, stream=None):
        """irr_extend_add of `level`'s Schur complements into their parents,
        one call per sibling round."""
        for r in self.rounds[level]:
            irr.irr_extend_add(r["batch"], r["max_n2"], r["n2"], r["F22"], r["ld22"], r["rel"], r["np_"],
                               r["Fp"], r["ldp"], r["info"], stream)

    def factor(self, stream=None):
        """The whole traversal, leaves to root (asynchronous on `stream`)."""
        for level in range(len(self.levels)):
            self.partial(level, stream)
            self.extend_add(level, stream)

    def extend_add_info(self):
        return [r["info"][: r["batch"]] for lvl in self.rounds for r in lvl]

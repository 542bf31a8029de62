"""Seeded synthetic inputs shared by the oracle side and the CUDA side.

This module holds NO arithmetic of the method (no elimination, no solve, no
update).  It only draws sizes and values, and builds structured test matrices
from factors that are *chosen* here (A = P*L*U is assembled by a plain product
of the chosen factors, which is input construction, not factorization).

Reference: sizes and value distributions follow the paper's workloads
(§V-A: "one thousand square matrices, whose sizes are randomly
sampled between 1 and the value shown on the x-axis") and the configs of
BASELINE.json / SURVEY.md §8(d).  The value generator is the counter-based
splitmix64 stream of SURVEY.md §8(d):

    a_ij = 2 * ((splitmix64(key + (i + j*m)) >> 11) * 2**-53) - 1
    key  = splitmix64(seed ^ splitmix64(global_id))

which is an exact dyadic in [-1, 1), independent of the leading dimension.
"""
from __future__ import annotations

import math
from dataclasses import dataclass

import numpy as np

__all__ = [
    "splitmix64", "matrix_key", "uniform_values", "hash_stream",
    "Config", "config", "CONFIG_NAMES",
    "g1_exact", "g1_singular", "g1_front", "g2_dominant",
    "front_values", "g1_front_lapack", "zuniform_values", "zg1_exact",
    "Tree", "assembly_tree", "tree_values", "tree_exact",
]

_M64 = np.uint64(0xFFFFFFFFFFFFFFFF)
_GOLD = np.uint64(0x9E3779B97F4A7C15)
_C1 = np.uint64(0xBF58476D1CE4E5B9)
_C2 = np.uint64(0x94D049BB133111EB)
_SALT = np.uint64(0xD1B54A32D192ED03)


def splitmix64(x):
    """Standard splitmix64 finalizer, all arithmetic mod 2**64."""
    with np.errstate(over="ignore"):
        z = np.asarray(x, dtype=np.uint64) + _GOLD
        z = (z ^ (z >> np.uint64(30))) * _C1
        z = (z ^ (z >> np.uint64(27))) * _C2
        return z ^ (z >> np.uint64(31))


def matrix_key(seed: int, gid, salt: int = 0):
    """Per-matrix stream key. salt=0 is the value stream of SURVEY §8(d);
    other salts give independent streams for the structured families."""
    with np.errstate(over="ignore"):
        s = np.uint64(seed & 0xFFFFFFFFFFFFFFFF)
        if salt:
            s = s ^ (np.uint64(salt) * _SALT)
        return splitmix64(s ^ splitmix64(np.asarray(gid, dtype=np.uint64)))


def hash_stream(seed: int, gid: int, salt: int, count: int) -> np.ndarray:
    """`count` uint64 draws of the stream (seed, gid, salt)."""
    key = matrix_key(seed, gid, salt)
    with np.errstate(over="ignore"):
        return splitmix64(key + np.arange(count, dtype=np.uint64))


def uniform_values(seed: int, gid: int, m: int, n: int) -> np.ndarray:
    """m x n Fortran-ordered matrix with entries exact dyadics in [-1, 1)."""
    key = matrix_key(seed, gid)
    with np.errstate(over="ignore"):
        x = splitmix64(key + np.arange(m * n, dtype=np.uint64))
    u = (x >> np.uint64(11)).astype(np.float64) * (2.0 ** -53)
    return (2.0 * u - 1.0).reshape((n, m)).T.copy(order="F") if m * n else np.zeros((m, n), order="F")


def front_values(seed: int, gid: int, nf: int) -> np.ndarray:
    """A frontal matrix is one nf x nf block, values as above."""
    return uniform_values(seed, gid, nf, nf)


# --------------------------------------------------------------------------
# Workload configurations (BASELINE.json configs)
# --------------------------------------------------------------------------
@dataclass
class Config:
    name: str
    kind: str            # "getrf" or "partial"
    m: np.ndarray        # getrf: rows;  partial: n1
    n: np.ndarray        # getrf: cols;  partial: n2
    seed: int
    description: str


CONFIG_NAMES = ("C1", "C1big", "C2", "C3", "C4", "C5", "C5partial")


def _sizes_c4c5(rng, count, tail_lo, tail_hi, mid_frac, tail_frac, log_mid):
    r = rng.random(count)
    nf = rng.integers(1, 64, size=count)                                  # U{1..63}
    mid = r >= (1.0 - mid_frac - tail_frac)
    tail = r >= (1.0 - tail_frac)
    lm = np.floor(np.exp(rng.uniform(math.log(64), math.log(1025), size=count))).astype(np.int64)
    lm = np.clip(lm, 64, 1024)
    nf = np.where(mid, lm, nf)
    nf = np.where(tail, rng.integers(tail_lo, tail_hi + 1, size=count), nf)
    return nf.astype(np.int64)


def config(name: str, scale: float = 1.0) -> Config:
    """Return the seeded size lists of a workload.  `scale` < 1 keeps the size
    distribution and shrinks the count (for tests / bounded CPU samples)."""
    idx = {"C1": 1, "C1big": 11, "C2": 2, "C3": 3, "C4": 4, "C5": 5, "C5partial": 5}[name]
    rng = np.random.Generator(np.random.PCG64(1000 + idx))
    seed = 1000 + idx
    if name == "C1":
        cnt = max(1, int(100 * scale))
        n = rng.integers(1, 33, size=cnt)
        return Config(name, "getrf", n.copy(), n.copy(), seed, "100 square FP64, n~U{1..32}")
    if name == "C1big":
        cnt = max(1, int(1048576 * scale))
        n = rng.integers(1, 33, size=cnt)
        return Config(name, "getrf", n.copy(), n.copy(), seed, "1,048,576 square FP64, n~U{1..32}")
    if name == "C2":
        cnt = max(1, int(10000 * scale))
        m = rng.integers(1, 257, size=cnt)
        n = rng.integers(1, 257, size=cnt)
        n[0::2] = m[0::2]                       # even i: square
        odd = np.arange(cnt) % 2 == 1
        while True:                             # odd i: resample n while n == m
            bad = odd & (n == m)
            if not bad.any():
                break
            n[bad] = rng.integers(1, 257, size=int(bad.sum()))
        return Config(name, "getrf", m, n, seed, "10,000 FP64, dims~U{1..256}, even square / odd rectangular m!=n")
    if name == "C3":
        cnt = max(1, int(2000 * scale))
        n = rng.integers(256, 1025, size=cnt)
        return Config(name, "getrf", n.copy(), n.copy(), seed, "2,000 square FP64, n~U{256..1024}")
    if name == "C4":
        cnt = max(1, int(50000 * scale))
        nf = _sizes_c4c5(rng, cnt, 3072, 4096, 0.099, 0.001, True)
        f = rng.uniform(0.25, 0.5, size=cnt)
        n1 = np.maximum(1, np.rint(f * nf)).astype(np.int64)
        n2 = nf - n1
        return Config(name, "partial", n1, n2, seed,
                      "50,000 fronts (90% U{1..63}, 9.9% log-U[64,1024], 0.1% U{3072..4096}); n1=rint(f*nf), f~U[.25,.5]")
    if name in ("C5", "C5partial"):
        cnt = max(1, int(200000 * scale))
        nf = _sizes_c4c5(rng, cnt, 1024, 2048, 0.09, 0.01, True)
        if name == "C5":
            return Config(name, "getrf", nf.copy(), nf.copy(), seed,
                          "200,000 fronts (90% U{1..63}, 9% log-U[64,1024], 1% U{1024..2048}), full DGETRF")
        f = rng.uniform(0.25, 0.5, size=cnt)
        n1 = np.maximum(1, np.rint(f * nf)).astype(np.int64)
        return Config(name, "partial", n1, nf - n1, seed, "C5 fronts, partial factorization (C4 rule)")
    raise KeyError(name)


# --------------------------------------------------------------------------
# Structured families (SURVEY.md §8(c) "Input families").  Each returns the
# matrix AND the factors it was assembled from; the expected outputs are the
# chosen factors, not the result of any elimination.
# --------------------------------------------------------------------------
_L_SET = np.array([0.0, 0.25, -0.25, 0.5, -0.5])
_UD_SET = np.array([1.0, -1.0, 2.0, -2.0])


def _apply_swaps_reverse(LU: np.ndarray, ipiv0: np.ndarray) -> np.ndarray:
    """A = S_0 S_1 ... S_{k-1} (LU): apply row interchanges k-1..0 (input assembly)."""
    A = LU.copy(order="F")
    for k in range(len(ipiv0) - 1, -1, -1):
        p = int(ipiv0[k])
        if p != k:
            A[[k, p], :] = A[[p, k], :]
    return A


def g1_exact(seed: int, gid: int, m: int, n: int, singular_col: int | None = None):
    """G1: exact dyadic family.  L unit lower (m x k) with off-diagonals in
    {0, +-1/4, +-1/2}; U (k x n) upper with integer off-diagonals in [-8, 8] and
    diagonal in {+-1, +-2}; 0-based ipiv[k] ~ U[k, m).  Returns
    (A, L, U, ipiv1based, info).  With singular_col=c (G1-sing): row c of U is
    zeroed, L(c+1:, c) = 0 and ipiv[c] = c, so info = c+1."""
    k = min(m, n)
    h = hash_stream(seed, gid, 1, m * k + k * n + k + 1)
    hl = h[: m * k].reshape((k, m)).T
    hu = h[m * k: m * k + k * n].reshape((n, k)).T
    hp = h[m * k + k * n:]
    L = np.zeros((m, k))
    for j in range(k):
        L[j, j] = 1.0
        idx = (hl[j + 1:, j] % np.uint64(len(_L_SET))).astype(np.int64)
        L[j + 1:, j] = _L_SET[idx]
    U = np.zeros((k, n))
    for i in range(k):
        U[i, i] = _UD_SET[int(hu[i, i] % np.uint64(4))]
        U[i, i + 1:] = (hu[i, i + 1:] % np.uint64(17)).astype(np.int64) - 8
    ipiv0 = np.array([j + int(hp[j] % np.uint64(m - j)) for j in range(k)], dtype=np.int64)
    info = 0
    if singular_col is not None:
        c = singular_col
        assert 0 <= c < k
        U[c, c:] = 0.0
        L[c + 1:, c] = 0.0
        ipiv0[c] = c
        info = c + 1
    LU = L @ U                 # exact: dyadic products, |entries| << 2**53
    A = _apply_swaps_reverse(LU, ipiv0)
    return np.asfortranarray(A), L, U, (ipiv0 + 1).astype(np.int32), info


def g1_singular(seed: int, gid: int, m: int, n: int, c: int):
    return g1_exact(seed, gid, m, n, singular_col=c)


def g1_front(seed: int, gid: int, n1: int, n2: int):
    """G1': exact dyadic front.  F11 from G1; X (n1 x n2), F21 (n2 x n1) and
    S (n2 x n2) small integers; F12 = F11 X, F22 = S + F21 X.  The partial
    factorization must return F12 -> X and F22 -> S exactly."""
    F11, L, U, ipiv, _ = g1_exact(seed, gid, n1, n1)
    h = hash_stream(seed, gid, 2, n1 * n2 * 2 + n2 * n2)
    X = ((h[: n1 * n2] % np.uint64(9)).astype(np.int64) - 4).astype(np.float64).reshape((n2, n1)).T
    F21 = ((h[n1 * n2: 2 * n1 * n2] % np.uint64(9)).astype(np.int64) - 4).astype(np.float64).reshape((n1, n2)).T
    S = ((h[2 * n1 * n2:] % np.uint64(9)).astype(np.int64) - 4).astype(np.float64).reshape((n2, n2)).T
    F12 = F11 @ X
    F22 = S + F21 @ X
    f = np.asfortranarray
    return dict(F11=f(F11), F12=f(F12), F21=f(F21), F22=f(F22), X=f(X), S=f(S), L=L, U=U, ipiv=ipiv)


def g1_front_lapack(seed: int, gid: int, n1: int, n2: int):
    """G1'' (LAPACK-style partial): F11 = P L U from G1;
    U12 = X (n1 x n2 small integers), L21 = Y (n2 x n1, entries in
    {0, +-1/4, +-1/2}), S (n2 x n2 small integers); F12 = P (L X),
    F21 = Y U, F22 = S + Y X (all exact).  The LAPACK-style partial
    factorization must return F12 -> X, F21 -> Y, F22 -> S exactly."""
    F11, L, U, ipiv, _ = g1_exact(seed, gid, n1, n1)
    h = hash_stream(seed, gid, 4, n1 * n2 * 2 + n2 * n2)
    X = ((h[: n1 * n2] % np.uint64(9)).astype(np.int64) - 4).astype(np.float64).reshape((n2, n1)).T
    Y = _L_SET[(h[n1 * n2: 2 * n1 * n2] % np.uint64(len(_L_SET))).astype(np.int64)].reshape((n1, n2)).T
    S = ((h[2 * n1 * n2:] % np.uint64(9)).astype(np.int64) - 4).astype(np.float64).reshape((n2, n2)).T
    F12 = _apply_swaps_reverse(L @ X, ipiv - 1) if n1 else np.zeros((0, n2))
    F21 = Y @ U
    F22 = S + Y @ X
    f = np.asfortranarray
    return dict(F11=f(F11), F12=f(F12), F21=f(F21), F22=f(F22), X=f(X), Y=f(Y), S=f(S), L=L, U=U, ipiv=ipiv)


# complex families (ZGETRF)
_ZL_SET = np.array([0, 0.25, -0.25, 0.5, -0.5, 0.25j, -0.25j, 0.5j, -0.5j, 0.25 + 0.25j, 0.25 - 0.25j,
                    -0.25 + 0.25j, -0.25 - 0.25j])
_ZUD_SET = np.array([1, -1, 2, -2, 1j, -1j, 2j, -2j])


def zuniform_values(seed: int, gid: int, m: int, n: int) -> np.ndarray:
    """m x n complex128 Fortran matrix: element e = i + j m takes its real part
    from draw 2e and its imaginary part from draw 2e+1 of the value stream
    (each an exact dyadic in [-1, 1), as uniform_values)."""
    key = matrix_key(seed, gid)
    with np.errstate(over="ignore"):
        x = splitmix64(key + np.arange(2 * m * n, dtype=np.uint64))
    u = 2.0 * ((x >> np.uint64(11)).astype(np.float64) * (2.0 ** -53)) - 1.0
    z = u[0::2] + 1j * u[1::2]
    return z.reshape((n, m)).T.copy(order="F") if m * n else np.zeros((m, n), dtype=np.complex128, order="F")


def zg1_exact(seed: int, gid: int, m: int, n: int, singular_col: int | None = None):
    """Complex G1: L unit lower with off-diagonals in {0, +-1/4, +-1/2, +-i/4,
    +-i/2, (+-1 +-i)/4} (|Re| + |Im| <= 1/2), U upper with Gaussian-integer
    off-diagonals in [-8, 8] + [-8, 8] i and diagonal in {+-1, +-2, +-i, +-2i},
    ipiv[k] ~ U[k, m).  Every candidate below the chosen pivot has at most
    half its |Re| + |Im|, every division is by a unit times 1 or 2 and every
    product is a Gaussian dyadic, so any correct complex GEPP with izamax
    pivoting returns L, U, ipiv bit-exactly.  Returns (A, L, U, ipiv, info)."""
    k = min(m, n)
    h = hash_stream(seed, gid, 5, m * k + 2 * k * n + k + 1)
    hl = h[: m * k].reshape((k, m)).T
    hu = h[m * k: m * k + 2 * k * n].reshape((2 * n, k)).T
    hp = h[m * k + 2 * k * n:]
    L = np.zeros((m, k), dtype=np.complex128)
    for j in range(k):
        L[j, j] = 1.0
        L[j + 1:, j] = _ZL_SET[(hl[j + 1:, j] % np.uint64(len(_ZL_SET))).astype(np.int64)]
    U = np.zeros((k, n), dtype=np.complex128)
    for i in range(k):
        U[i, i] = _ZUD_SET[int(hu[i, i] % np.uint64(8))]
        re = (hu[i, i + 1:n] % np.uint64(17)).astype(np.int64) - 8
        im = (hu[i, n + i + 1:2 * n] % np.uint64(17)).astype(np.int64) - 8
        U[i, i + 1:] = re + 1j * im
    ipiv0 = np.array([j + int(hp[j] % np.uint64(m - j)) for j in range(k)], dtype=np.int64)
    info = 0
    if singular_col is not None:
        c = singular_col
        U[c, c:] = 0.0
        L[c + 1:, c] = 0.0
        ipiv0[c] = c
        info = c + 1
    A = _apply_swaps_reverse(L @ U, ipiv0)
    return np.asfortranarray(A), L, U, (ipiv0 + 1).astype(np.int32), info


def g2_dominant(seed: int, gid: int, m: int, n: int):
    """G2: permuted column-diagonally-dominant matrix.  Off-diagonals U[-1,1);
    for j < k: a_jj = +-(2*sum_{i!=j}|a_ij| + 1); rows permuted by pi (row r
    holds original row pi[r]).  Returns (A, ipiv1based) where ipiv follows from
    pi alone: cur = pi; for each j, ipiv[j] = position of j in cur; swap."""
    k = min(m, n)
    B = uniform_values(seed, gid, m, n).copy()
    h = hash_stream(seed, gid, 3, m + k)
    for j in range(k):
        col = np.abs(B[:, j]).sum() - abs(B[j, j])
        sgn = 1.0 if (h[m + j] & np.uint64(1)) else -1.0
        B[j, j] = sgn * (2.0 * col + 1.0)
    pi = np.arange(m)
    for t in range(m - 1, 0, -1):            # Fisher-Yates on the hash stream
        r = int(h[t] % np.uint64(t + 1))
        pi[t], pi[r] = pi[r], pi[t]
    A = np.asfortranarray(B[pi, :])
    cur = list(pi)
    ipiv = np.zeros(k, dtype=np.int32)
    for j in range(k):
        p = cur.index(j, j)
        ipiv[j] = p + 1
        cur[j], cur[p] = cur[p], cur[j]
    return A, ipiv


# --------------------------------------------------------------------------
# Packed batches: every matrix's values written straight into one flat
# column-major buffer (matrix g at offsets[g], leading dimension ld[g]).
# --------------------------------------------------------------------------
def packed_offsets(ld, n, align: int = 32):
    """Element offsets of each matrix in a flat buffer, starts aligned to
    `align` elements (32 doubles = 256 B).  Returns (offsets, total)."""
    ld = np.asarray(ld, dtype=np.int64)
    n = np.asarray(n, dtype=np.int64)
    sizes = ((ld * n + align - 1) // align) * align
    offsets = np.zeros(len(sizes), dtype=np.int64)
    if len(sizes) > 1:
        np.cumsum(sizes[:-1], out=offsets[1:])
    total = int(offsets[-1] + sizes[-1]) if len(sizes) else 0
    return offsets, max(total, align)


def fill_packed(seed: int, m, n, ld, offsets, out: np.ndarray, gid_base: int = 0, chunk: int = 1 << 24,
                gids=None):
    """Write uniform_values(seed, gid(g), m[g], n[g]) for every g into
    out[offsets[g] + i + j*ld[g]] (vectorised over matrices, chunked), where
    gid(g) = gids[g] if given, else gid_base + g."""
    gid_of = (np.arange(len(m), dtype=np.int64) + gid_base) if gids is None else np.asarray(gids, dtype=np.int64)
    m = np.asarray(m, dtype=np.int64)
    n = np.asarray(n, dtype=np.int64)
    ld = np.asarray(ld, dtype=np.int64)
    offsets = np.asarray(offsets, dtype=np.int64)
    cnt = m * n
    g0 = 0
    B = len(m)
    while g0 < B:
        # take matrices until ~chunk elements
        csum = np.cumsum(cnt[g0:])
        g1 = g0 + int(np.searchsorted(csum, chunk, side="right")) + 1
        g1 = min(max(g1, g0 + 1), B)
        gs = np.arange(g0, g1)
        c = cnt[gs]
        tot = int(c.sum())
        if tot:
            gid = np.repeat(gs, c)
            starts = np.repeat(np.cumsum(c) - c, c)
            e = np.arange(tot, dtype=np.int64) - starts           # i + j*m
            keys = matrix_key(seed, gid_of[gid].astype(np.uint64))
            with np.errstate(over="ignore"):
                x = splitmix64(keys + e.astype(np.uint64))
            vals = 2.0 * ((x >> np.uint64(11)).astype(np.float64) * (2.0 ** -53)) - 1.0
            mm = m[gid]
            j = e // np.maximum(mm, 1)
            i = e - j * mm
            out[offsets[gid] + i + j * ld[gid]] = vals
        g0 = g1
    return out


def extend_add_level(seed: int, n_parents: int, np_max: int, children_per_parent: int = 2,
                     frac_lo: float = 0.25, frac_hi: float = 0.75):
    """One level of a synthetic binary assembly tree for the extend-add.

    Parent p has order np_p ~ U[1, np_max]; each of its children has a Schur
    complement of order n2_c ~ U[frac_lo, frac_hi] * np_p (at least 1, at most
    np_p) whose rows / columns map to a sorted random subset rel_c of the
    parent's indices (nested dissection: a child's separator variables appear
    in its parent front, in order).  Children are listed parent by parent
    (child 0 of parent 0, child 1 of parent 0, ...).  Values from
    uniform_values.  Returns (np_sizes, parent_of_child, n2, rel list,
    F22 list, Fp list) -- no arithmetic of the method.
    """
    rng = np.random.default_rng(seed)
    np_sizes = rng.integers(1, np_max + 1, size=n_parents).astype(np.int32)
    parent, n2, rel, F22 = [], [], [], []
    Fp = [uniform_values(seed, 1_000_000 + p, int(s), int(s)) for p, s in enumerate(np_sizes)]
    gid = 0
    for p, s in enumerate(np_sizes):
        for _ in range(children_per_parent):
            k = int(rng.integers(max(1, int(frac_lo * s)), max(1, int(frac_hi * s)) + 1))
            k = min(max(k, 1), int(s))
            r = np.sort(rng.choice(int(s), size=k, replace=False)).astype(np.int32)
            parent.append(p)
            n2.append(k)
            rel.append(r)
            F22.append(uniform_values(seed, gid, k, k))
            gid += 1
    return np_sizes, np.array(parent, dtype=np.int32), np.array(n2, dtype=np.int32), rel, F22, Fp


# --------------------------------------------------------------------------
# Synthetic assembly trees (§III-A):
# the tree is traversed level by level from the leaves to the root; each
# front F_r = [F11 F12; F21 F22] is partially factored and its Schur
# complement F22 is extend-added into the parent front through an index map.
# --------------------------------------------------------------------------
@dataclass
class Tree:
    n1: np.ndarray          # fully summed variables of each node (its separator)
    n2: np.ndarray          # contribution-block order (0 at the root)
    parent: np.ndarray      # parent node, -1 at the root
    rel: list               # rel[c]: int32[n2[c]], sorted rows / cols of the parent front
    levels: list            # node ids per level, leaves first (a node's parent is on a later level)

    @property
    def nf(self):
        return self.n1 + self.n2


def assembly_tree(seed: int, depth: int, s0: float = 8.0, growth: float = 1.41, cfrac=(0.4, 0.9)) -> Tree:
    """Complete binary tree of `depth` levels shaped like nested dissection of
    a 2-D grid: a node at height h (leaves h = 0) owns n1 ~ s0 growth^h
    U[0.75, 1.25] separator variables; a child's contribution block has
    n2_c ~ U[cfrac] * nf_parent variables, mapped to a sorted random subset of
    the parent front's nf_p = n1_p + n2_p indices.  Input construction only."""
    rng = np.random.default_rng(seed)
    nodes = 2 ** depth - 1
    # node ids: level by level from the leaves; level h holds 2^(depth-1-h) nodes
    levels, start = [], 0
    for h in range(depth):
        cnt = 2 ** (depth - 1 - h)
        levels.append(np.arange(start, start + cnt))
        start += cnt
    height = np.concatenate([np.full(len(l), h) for h, l in enumerate(levels)])
    n1 = np.maximum(1, np.rint(s0 * growth ** height * rng.uniform(0.75, 1.25, nodes))).astype(np.int64)
    parent = np.full(nodes, -1, dtype=np.int64)
    for h in range(depth - 1):
        parent[levels[h]] = levels[h + 1][np.arange(len(levels[h])) // 2]
    n2 = np.zeros(nodes, dtype=np.int64)
    rel = [np.zeros(0, dtype=np.int32) for _ in range(nodes)]
    for h in range(depth - 2, -1, -1):        # top down: the parent's front order is known
        for c in levels[h]:
            p = parent[c]
            nfp = int(n1[p] + n2[p])
            k = int(np.clip(np.rint(rng.uniform(*cfrac) * nfp), 1, nfp))
            n2[c] = k
            rel[c] = np.sort(rng.choice(nfp, size=k, replace=False)).astype(np.int32)
    return Tree(n1, n2, parent, rel, levels)


def tree_values(seed: int, tree: Tree):
    """Original front values (before any extend-add): uniform dyadics, one
    nf x nf block per node keyed by node id."""
    return [front_values(seed, int(v), int(tree.n1[v] + tree.n2[v])) for v in range(len(tree.n1))]


def tree_exact(seed: int, tree: Tree):
    """Exact dyadic tree: every node's ASSEMBLED front (original + the
    children's Schur complements) is a G1' front, so the partial factorization
    of every node returns its chosen factors bit-exactly: F11 -> L\\U (with the
    chosen ipiv), F12 -> X, F22 -> S.  The original of node p is the G1' front
    minus the extend-add of its children's chosen S_c (small integers; exact).
    Returns (originals, expected) with expected[v] = the g1_front dict."""
    exp = [g1_front(seed, int(v), int(tree.n1[v]), int(tree.n2[v])) for v in range(len(tree.n1))]
    orig = []
    for v in range(len(tree.n1)):
        e, a = exp[v], int(tree.n1[v])
        F = np.zeros((a + int(tree.n2[v]),) * 2, order="F")
        F[:a, :a], F[:a, a:], F[a:, :a], F[a:, a:] = e["F11"], e["F12"], e["F21"], e["F22"]
        orig.append(F)
    for c in range(len(tree.n1)):
        p = tree.parent[c]
        if p >= 0:
            r = tree.rel[c]
            orig[p][np.ix_(r, r)] -= exp[c]["S"]
    return orig, exp

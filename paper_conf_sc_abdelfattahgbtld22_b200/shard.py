"""Flop-balanced sharding of an irregular batch over the GPUs of one box
(north_star: "fronts are partitioned flop-balanced across the GPUs ... with
NCCL over NVLink used only to gather per-matrix info/pivot status").

Host-side bookkeeping only: the matrices are independent, so the only data-
path exchange is the final gather of the per-matrix status words.
"""
from __future__ import annotations

import heapq

import numpy as np


def lpt_partition(work, parts: int) -> np.ndarray:
    """Longest-processing-time-first greedy: items sorted by decreasing work,
    each given to the currently least-loaded part (ties -> lowest part id).
    Returns owner[i] in [0, parts).  Deterministic.  Computed by the C ABI's
    irr_shard_lpt_work (host code in libirr.so)."""
    from . import irr
    work = np.asarray(work, dtype=np.float64)
    if parts <= 1 or len(work) == 0:
        return np.zeros(len(work), dtype=np.int64)
    return irr.irr_shard_lpt_work(work, parts).astype(np.int64)


def lpt_partition_reference(work, parts: int) -> np.ndarray:
    """The same greedy in Python (tests compare the C ABI against it)."""
    work = np.asarray(work, dtype=np.float64)
    owner = np.zeros(len(work), dtype=np.int64)
    if parts <= 1 or len(work) == 0:
        return owner
    order = np.lexsort((np.arange(len(work)), -work))   # by work desc, then index asc
    heap = [(0.0, p) for p in range(parts)]
    heapq.heapify(heap)
    for i in order:
        load, p = heapq.heappop(heap)
        owner[i] = p
        heapq.heappush(heap, (load + work[i], p))
    return owner


def shard_indices(work, parts: int, rank: int) -> np.ndarray:
    """Global indices owned by `rank`, in ascending order."""
    return np.nonzero(lpt_partition(work, parts) == rank)[0]


def imbalance(work, owner, parts: int) -> float:
    """max part load / mean part load (1.0 = perfect)."""
    loads = np.bincount(owner, weights=np.asarray(work, dtype=np.float64), minlength=parts)
    mean = loads.mean()
    return float(loads.max() / mean) if mean > 0 else 1.0


def merge_status(gathered: np.ndarray, shards) -> np.ndarray:
    """Scatter the gathered per-rank status rows back to global order.
    gathered: [parts, pad] array (row r = rank r's status words, padded);
    shards: list of index arrays (rank r's global indices)."""
    total = sum(len(s) for s in shards)
    out = np.zeros(total, dtype=gathered.dtype)
    for r, idx in enumerate(shards):
        out[idx] = gathered[r, : len(idx)]
    return out


def sibling_rounds(parent_of_child) -> list:
    """Split one tree level's children into rounds for irr_extend_add:
    round r holds the r-th child (in batch order) of every parent, so no two
    children of one round share a parent and each call adds at most one
    contribution per parent entry (bit-identical to the sequential order,
    include/irr.h).  Returns a list of ascending index arrays."""
    parent = np.asarray(parent_of_child, dtype=np.int64)
    if len(parent) == 0:
        return []
    order = np.argsort(parent, kind="stable")
    ps = parent[order]
    first = np.r_[0, np.nonzero(np.diff(ps))[0] + 1]
    rank = np.arange(len(ps)) - np.repeat(first, np.diff(np.r_[first, len(ps)]))
    r_of = np.empty(len(parent), dtype=np.int64)
    r_of[order] = rank
    return [np.nonzero(r_of == r)[0] for r in range(int(r_of.max()) + 1)]


def shard_level(parent_of_child, n2, parts: int) -> np.ndarray:
    """Owner rank of each child of one extend-add level: a parent front and
    all its children stay on one GPU (the scatter needs no exchange), parents
    LPT-balanced by the bytes their children move (sum of n2^2)."""
    parent = np.asarray(parent_of_child, dtype=np.int64)
    if len(parent) == 0:
        return np.zeros(0, dtype=np.int64)
    n2 = np.asarray(n2, dtype=np.float64)
    work = np.bincount(parent, weights=n2 * n2)
    return lpt_partition(work, parts)[parent]

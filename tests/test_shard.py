"""Host logic of the multi-GPU path: LPT flop-balanced
partition and the status gather, exercised with world_size 2 over gloo on CPU."""
import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

import irrgen
from paper_conf_sc_abdelfattahgbtld22_b200 import flops as F
from paper_conf_sc_abdelfattahgbtld22_b200.shard import imbalance, lpt_partition, merge_status, shard_indices


def test_lpt_is_a_partition_and_balanced():
    cfg = irrgen.config("C5", scale=0.1)           # 20,000 fronts, heavy tail
    w = F.getrf_flops(cfg.m, cfg.n)
    for parts in (1, 2, 4, 8):
        owner = lpt_partition(w, parts)
        assert owner.min() >= 0 and owner.max() < parts
        shards = [shard_indices(w, parts, r) for r in range(parts)]
        allidx = np.sort(np.concatenate(shards))
        assert np.array_equal(allidx, np.arange(len(w)))
        assert imbalance(w, owner, parts) < 1.01
    # deterministic
    assert np.array_equal(lpt_partition(w, 8), lpt_partition(w, 8))


def test_lpt_small_cases():
    assert list(lpt_partition([5, 4, 3, 3, 3], 2)) == [0, 1, 1, 0, 1]   # loads 8 / 10 -> LPT greedy
    assert list(lpt_partition([], 3)) == []
    assert list(lpt_partition([1.0], 4)) == [0]


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _status_words(cfg, gids):
    """(info, FNV-1a of ipiv) per matrix -- the record irr_status_words
    writes on the GPU (include/irr.h; GPU test_status_words pins the GPU words
    to this host definition) -- here from the oracle's factorization."""
    import oracle
    from gpu_util import fnv1a_ipiv
    out = np.zeros((len(gids), 2), dtype=np.int64)
    for q, g in enumerate(gids):
        A = irrgen.uniform_values(cfg.seed, int(g), int(cfg.m[g]), int(cfg.n[g]))
        _, ip, info, _ = oracle.getrf(A)
        out[q] = (info, fnv1a_ipiv(ip))
    return out


def _worker(rank, world, port, q):
    import sys
    sys.path.insert(0, os.path.dirname(os.path.abspath(__file__)))
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    cfg = irrgen.config("C2", scale=0.02)          # the same 200 matrices at every world size (strong)
    w = F.getrf_flops(cfg.m, cfg.n)
    owner = lpt_partition(w, world)
    mine = np.nonzero(owner == rank)[0]
    pad = int(np.bincount(owner, minlength=world).max())
    # this rank's real status words (info, ipiv hash) of its own matrices, padded
    status = torch.full((pad, 2), -7, dtype=torch.int64)
    status[: len(mine)] = torch.from_numpy(_status_words(cfg, mine))
    gathered = torch.zeros(world * pad, 2, dtype=torch.int64)
    dist.all_gather_into_tensor(gathered, status)
    t = torch.tensor([float(rank + 1)], dtype=torch.float64)
    dist.all_reduce(t, op=dist.ReduceOp.MAX)       # max-over-ranks timing reduction
    if rank == 0:
        shards = [np.nonzero(owner == r)[0] for r in range(world)]
        g = gathered.view(world, pad, 2).numpy()
        merged = np.stack([merge_status(g[:, :, f], shards) for f in range(2)], axis=1)
        q.put((merged.tolist(), float(t.item()), len(w)))
    dist.destroy_process_group()


def test_gloo_two_ranks_gather_and_merge():
    """world_size 2 over gloo: every matrix's status word lands at its global
    id after the gather, and the gathered words equal the single-process
    (G = 1) words bitwise (results independent of G)."""
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, 2, port, q)) for r in range(2)]
    for p in procs:
        p.start()
    merged, tmax, total = q.get(timeout=300)
    for p in procs:
        p.join(timeout=60)
        assert p.exitcode == 0
    cfg = irrgen.config("C2", scale=0.02)
    import sys
    sys.path.insert(0, os.path.dirname(os.path.abspath(__file__)))
    single = _status_words(cfg, np.arange(total))
    assert np.array_equal(np.array(merged), single)
    assert tmax == 2.0


def test_lpt_c_abi_equals_reference():
    """irr_shard_lpt_work (C ABI, host) == the Python LPT greedy, and
    irr_shard_lpt (flops from m, n) == irr_shard_lpt_work on FLOPS_DGETRF."""
    from paper_conf_sc_abdelfattahgbtld22_b200 import irr
    from paper_conf_sc_abdelfattahgbtld22_b200.shard import lpt_partition_reference
    cfg = irrgen.config("C5", scale=0.05)
    w = F.getrf_flops(cfg.m, cfg.n)
    for parts in (2, 3, 8):
        assert np.array_equal(lpt_partition(w, parts), lpt_partition_reference(w, parts))
        m32 = np.ascontiguousarray(cfg.m, dtype=np.int32)
        n32 = np.ascontiguousarray(cfg.n, dtype=np.int32)
        owner = np.zeros(len(w), dtype=np.int32)
        assert irr.load().irr_shard_lpt(len(w), m32.ctypes.data, n32.ctypes.data, parts, owner.ctypes.data) == 0
        assert np.array_equal(owner, lpt_partition(w, parts))


def test_sibling_rounds_and_level_shard():
    from paper_conf_sc_abdelfattahgbtld22_b200.shard import shard_level, sibling_rounds
    import irrgen
    nps, parent, n2, rel, F22, Fp = irrgen.extend_add_level(2, 50, 64, children_per_parent=3)
    perm = np.random.default_rng(0).permutation(len(parent))      # children in any order
    parent, n2 = parent[perm], n2[perm]
    rounds = sibling_rounds(parent)
    assert len(rounds) == 3
    assert sorted(np.concatenate(rounds).tolist()) == list(range(len(parent)))
    for r in rounds:
        assert len(np.unique(parent[r])) == len(r)                 # no shared parent in a round
    # round r holds the r-th occurrence of each parent in batch order
    for c in range(len(parent)):
        k = int((parent[:c] == parent[c]).sum())
        assert c in rounds[k]
    owner = shard_level(parent, n2, 4)
    for p in np.unique(parent):
        assert len(np.unique(owner[parent == p])) == 1              # a parent and its children on one rank
    assert sibling_rounds([]) == [] and len(shard_level([], [], 2)) == 0

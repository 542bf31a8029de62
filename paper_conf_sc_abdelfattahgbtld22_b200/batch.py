"""Caller-side device storage for irregular batches (setup, not the method).

The C ABI takes caller-owned device pointer arrays ("the array of
pointers must exist in the GPU memory before the kernel is launched").  These
helpers lay a batch out once in HBM and build those arrays:

  * MatrixBatch: one flat float64 buffer, matrix i column-major with leading
    dimension ld[i], every matrix starting on a 256-byte boundary; a flat int32
    ipiv buffer; info[batch]; int32 size arrays; int64 pointer arrays.
  * FrontBatch: one nf x nf block per front (ld = nf) with the four pointer
    arrays F11 / F12 / F21 / F22 into it (SURVEY §8(d) C4 layout).

Only torch is used here, for device memory and copies.
"""
from __future__ import annotations

import numpy as np
import torch

from . import irr

ALIGN = 32  # elements (256 B)


def _offsets(sizes: np.ndarray, align: int = ALIGN):
    sizes = ((np.asarray(sizes, dtype=np.int64) + align - 1) // align) * align
    off = np.zeros(len(sizes), dtype=np.int64)
    if len(sizes) > 1:
        np.cumsum(sizes[:-1], out=off[1:])
    total = int(off[-1] + sizes[-1]) if len(sizes) else 0
    return off, max(total, align)


class MatrixBatch:
    def __init__(self, m, n, ld=None, device="cuda", with_ipiv=True, data=None):
        """data: optional existing float64 buffer (>= total elements) to lay
        the batch out in (e.g. a prefix of a larger batch), else allocated."""
        self.m_h = np.asarray(m, dtype=np.int64)
        self.n_h = np.asarray(n, dtype=np.int64)
        self.batch = len(self.m_h)
        self.ld_h = np.maximum(1, self.m_h) if ld is None else np.asarray(ld, dtype=np.int64)
        self.device = torch.device(device) if data is None else data.device
        self.offsets, self.total = _offsets(self.ld_h * self.n_h)
        if data is None:
            self.data = torch.empty(self.total, dtype=torch.float64, device=self.device)
        else:
            assert data.dtype == torch.float64 and data.numel() >= self.total
            self.data = data[: self.total]
        base = self.data.data_ptr()
        self.ptr = torch.from_numpy(base + 8 * self.offsets).to(self.device)
        self.m = torch.from_numpy(self.m_h.astype(np.int32)).to(self.device)
        self.n = torch.from_numpy(self.n_h.astype(np.int32)).to(self.device)
        self.ld = torch.from_numpy(self.ld_h.astype(np.int32)).to(self.device)
        self.max_m = int(self.m_h.max()) if self.batch else 0
        self.max_n = int(self.n_h.max()) if self.batch else 0
        self.k_h = np.minimum(self.m_h, self.n_h)
        if with_ipiv:
            self.ipiv_off, ipiv_total = _offsets(self.k_h)
            self.ipiv_data = torch.zeros(ipiv_total, dtype=torch.int32, device=self.device)
            self.ipiv = torch.from_numpy(self.ipiv_data.data_ptr() + 4 * self.ipiv_off).to(self.device)
        self.info = torch.zeros(max(1, self.batch), dtype=torch.int32, device=self.device)
        self.work = None

    # -- host <-> device (setup / verification helpers)
    def host_buffer(self, pinned=False):
        return torch.empty(self.total, dtype=torch.float64, pin_memory=pinned)

    def matrix(self, i, flat_host: np.ndarray):
        """View of matrix i (m x n, Fortran) inside a flat host copy of data."""
        o, m, n, ld = int(self.offsets[i]), int(self.m_h[i]), int(self.n_h[i]), int(self.ld_h[i])
        if m * n == 0:
            return np.zeros((m, n), order="F")
        return np.lib.stride_tricks.as_strided(flat_host[o:], shape=(m, n), strides=(8, 8 * ld))

    def ipiv_of(self, i, ipiv_host: np.ndarray):
        o, k = int(self.ipiv_off[i]), int(self.k_h[i])
        return ipiv_host[o:o + k]

    def workspace(self):
        if self.work is None:
            nb = irr.irr_getrf_workspace_size(self.batch, self.max_m, self.max_n)
            self.work = torch.empty(max(256, nb), dtype=torch.uint8, device=self.device)
        return self.work

    def getrf(self, stream=None, max_m=None, max_n=None):
        """irr_getrf on the whole batch (asynchronous on `stream`)."""
        return irr.irr_getrf(self.batch, self.max_m if max_m is None else max_m,
                             self.max_n if max_n is None else max_n, self.m, self.n, self.ptr, self.ld,
                             self.ipiv, self.info, self.workspace(), stream)


    def getrs(self, rhs: "MatrixBatch", info=None, stream=None):
        """irr_getrs: rhs.data[i] <- A_i^-1 rhs_i with this batch's factors
        (square matrices; rhs.m must equal this batch's n).  Returns the
        per-system argument status (int32 device tensor)."""
        if info is None:
            info = torch.zeros(max(1, self.batch), dtype=torch.int32, device=self.device)
        nb = irr.irr_getrs_workspace_size(self.batch)
        work = torch.empty(max(256, nb), dtype=torch.uint8, device=self.device)
        irr.irr_getrs(irr.IRR_NO_TRANS, self.batch, self.max_n, rhs.max_n, self.n, rhs.n, self.ptr, self.ld,
                      self.ipiv, rhs.ptr, rhs.ld, info, work, stream)
        self._getrs_keep = work
        return info


class FrontBatch:
    """Fronts F = [F11 F12; F21 F22], one nf x nf block each (ld = nf)."""

    def __init__(self, n1, n2, device="cuda"):
        self.n1_h = np.asarray(n1, dtype=np.int64)
        self.n2_h = np.asarray(n2, dtype=np.int64)
        self.nf_h = self.n1_h + self.n2_h
        self.batch = len(self.n1_h)
        self.device = torch.device(device)
        ldf = np.maximum(1, self.nf_h)
        self.ld_h = ldf
        self.offsets, self.total = _offsets(ldf * self.nf_h)
        self.data = torch.empty(self.total, dtype=torch.float64, device=self.device)
        base = self.data.data_ptr() + 8 * self.offsets
        nf, a = self.nf_h, self.n1_h

        def P(x):
            return torch.from_numpy(np.asarray(x, dtype=np.int64)).to(self.device)

        self.F11 = P(base)
        self.F12 = P(base + 8 * a * ldf)
        self.F21 = P(base + 8 * a)
        self.F22 = P(base + 8 * (a + a * ldf))
        ld32 = torch.from_numpy(ldf.astype(np.int32)).to(self.device)
        self.ld11 = self.ld12 = self.ld21 = self.ld22 = ld32
        self.n1 = torch.from_numpy(self.n1_h.astype(np.int32)).to(self.device)
        self.n2 = torch.from_numpy(self.n2_h.astype(np.int32)).to(self.device)
        self.max_n1 = int(self.n1_h.max()) if self.batch else 0
        self.max_n2 = int(self.n2_h.max()) if self.batch else 0
        self.ipiv_off, ipiv_total = _offsets(self.n1_h)
        self.ipiv_data = torch.zeros(ipiv_total, dtype=torch.int32, device=self.device)
        self.ipiv = P(self.ipiv_data.data_ptr() + 4 * self.ipiv_off)
        self.info = torch.zeros(max(1, self.batch), dtype=torch.int32, device=self.device)
        self.work = None

    def front(self, i, flat_host: np.ndarray):
        o, nf = int(self.offsets[i]), int(self.nf_h[i])
        if nf == 0:
            return np.zeros((0, 0), order="F")
        return np.lib.stride_tricks.as_strided(flat_host[o:], shape=(nf, nf), strides=(8, 8 * max(1, nf)))

    def ipiv_of(self, i, ipiv_host: np.ndarray):
        o, k = int(self.ipiv_off[i]), int(self.n1_h[i])
        return ipiv_host[o:o + k]

    def workspace(self):
        if self.work is None:
            nb = irr.irr_getrf_partial_workspace_size(self.batch, self.max_n1, self.max_n2)
            self.work = torch.empty(max(256, nb), dtype=torch.uint8, device=self.device)
        return self.work

    def getrf_partial(self, stream=None, lapack=False):
        """irr_getrf_partial (the paper's steps), or with lapack=True
        irr_getrf_partial_lapack (F12 -> U12, F21 -> L21)."""
        fn = irr.irr_getrf_partial_lapack if lapack else irr.irr_getrf_partial
        return fn(self.batch, self.max_n1, self.max_n2, self.n1, self.n2, self.F11, self.ld11, self.F12, self.ld12,
                  self.F21, self.ld21, self.F22, self.ld22, self.ipiv, self.info, self.workspace(), stream)


# ---------------------------------------------------------------------------
# End to end with HOST buffers: the batch is streamed through the GPU in
# contiguous chunks of matrices, so the host->device copy of chunk c+1, the
# factorization of chunk c and the device->host copy of chunk c-1 overlap (two
# copy streams -- B200 has copy engines in both directions -- and one compute
# stream; every library call stays on the compute stream, so the library's
# own forked side stream is never shared by two concurrent calls).  Matrices
# are independent, so a chunk is just a sub-batch: views of the size / pointer
# / ipiv / info arrays at an offset, no copies.
# ---------------------------------------------------------------------------
def _chunk_bounds(offsets, total, count, chunks):
    """Matrix index boundaries splitting the flat buffer into ~equal byte ranges."""
    if count == 0:
        return [0, 0]
    chunks = max(1, min(chunks, count))
    ends = np.append(np.asarray(offsets[1:], dtype=np.int64), total)
    cuts = [0]
    for c in range(1, chunks):
        i = int(np.searchsorted(ends, total * c / chunks, side="left")) + 1
        if cuts[-1] < i < count:
            cuts.append(i)
    cuts.append(count)
    return cuts


class _Pipe:
    def __init__(self, device):
        self.h2d = torch.cuda.Stream(device)
        self.d2h = torch.cuda.Stream(device)

    def run(self, cuts, elem_range, data, host_in, host_out, compute, extra_out):
        """elem_range(i0, i1) -> (e0, e1) flat element range of matrices [i0, i1);
        compute(i0, i1, stream) factors that sub-batch; extra_out: list of
        (device tensor, host tensor, range_fn) copied back per chunk."""
        cur = torch.cuda.current_stream(data.device)
        self.h2d.wait_stream(cur)
        self.d2h.wait_stream(cur)
        loaded, done = [], []
        for i0, i1 in zip(cuts[:-1], cuts[1:]):
            e0, e1 = elem_range(i0, i1)
            with torch.cuda.stream(self.h2d):
                data[e0:e1].copy_(host_in[e0:e1], non_blocking=True)
                ev = torch.cuda.Event()
                ev.record(self.h2d)
            loaded.append(ev)
        for (i0, i1), ev in zip(zip(cuts[:-1], cuts[1:]), loaded):
            cur.wait_event(ev)
            compute(i0, i1, cur)
            evc = torch.cuda.Event()
            evc.record(cur)
            done.append(evc)
        for (i0, i1), evc in zip(zip(cuts[:-1], cuts[1:]), done):
            self.d2h.wait_event(evc)
            e0, e1 = elem_range(i0, i1)
            with torch.cuda.stream(self.d2h):
                host_out[e0:e1].copy_(data[e0:e1], non_blocking=True)
                for dev_t, host_t, rng in extra_out:
                    a, b = rng(i0, i1)
                    host_t[a:b].copy_(dev_t[a:b], non_blocking=True)
        cur.wait_stream(self.d2h)


def _sub(t, i0, i1):
    return t[i0:i1]


def getrf_host(B: "MatrixBatch", host_in, host_out, ipiv_out, info_out, chunks=8, pipe=None):
    """irr_getrf end to end from pinned host buffers (flat layout of B):
    host_out <- factors, ipiv_out <- pivots (flat), info_out <- info.  Ordered
    on torch's current stream (the caller synchronises to read the results)."""
    pipe = pipe or _Pipe(B.device)
    cuts = _chunk_bounds(B.offsets, B.total, B.batch, chunks)
    ends = np.append(B.offsets[1:], B.total) if B.batch else np.zeros(0, dtype=np.int64)
    pends = np.append(B.ipiv_off[1:], B.ipiv_data.numel()) if B.batch else np.zeros(0, dtype=np.int64)

    def rng(i0, i1):
        return int(B.offsets[i0]), int(ends[i1 - 1])

    def prng(i0, i1):
        return int(B.ipiv_off[i0]), int(pends[i1 - 1])

    def compute(i0, i1, s):
        irr.irr_getrf(i1 - i0, int(B.m_h[i0:i1].max()), int(B.n_h[i0:i1].max()), _sub(B.m, i0, i1),
                      _sub(B.n, i0, i1), _sub(B.ptr, i0, i1), _sub(B.ld, i0, i1), _sub(B.ipiv, i0, i1),
                      _sub(B.info, i0, i1), B.workspace(), s)

    pipe.run(cuts, rng, B.data, host_in, host_out, compute,
             [(B.ipiv_data, ipiv_out, prng), (B.info, info_out, lambda a, b: (a, b))])
    return pipe


def getrf_partial_host(F: "FrontBatch", host_in, host_out, ipiv_out, info_out, chunks=8, pipe=None):
    """irr_getrf_partial end to end from pinned host buffers (flat layout of F)."""
    pipe = pipe or _Pipe(F.device)
    cuts = _chunk_bounds(F.offsets, F.total, F.batch, chunks)
    ends = np.append(F.offsets[1:], F.total) if F.batch else np.zeros(0, dtype=np.int64)
    pends = np.append(F.ipiv_off[1:], F.ipiv_data.numel()) if F.batch else np.zeros(0, dtype=np.int64)

    def rng(i0, i1):
        return int(F.offsets[i0]), int(ends[i1 - 1])

    def prng(i0, i1):
        return int(F.ipiv_off[i0]), int(pends[i1 - 1])

    def compute(i0, i1, s):
        S = lambda t: _sub(t, i0, i1)  # noqa: E731
        irr.irr_getrf_partial(i1 - i0, int(F.n1_h[i0:i1].max()), int(F.n2_h[i0:i1].max()), S(F.n1), S(F.n2),
                              S(F.F11), S(F.ld11), S(F.F12), S(F.ld12), S(F.F21), S(F.ld21), S(F.F22),
                              S(F.ld22), S(F.ipiv), S(F.info), F.workspace(), s)

    pipe.run(cuts, rng, F.data, host_in, host_out, compute,
             [(F.ipiv_data, ipiv_out, prng), (F.info, info_out, lambda a, b: (a, b))])
    return pipe


class ZMatrixBatch:
    """Complex batch for irr_zgetrf: matrix i is m x n complex (interleaved
    re / im doubles), column-major with ld[i] complex elements, starting on a
    256-byte boundary; int32 ipiv buffer, info, size and pointer arrays."""

    def __init__(self, m, n, ld=None, device="cuda"):
        self.m_h = np.asarray(m, dtype=np.int64)
        self.n_h = np.asarray(n, dtype=np.int64)
        self.batch = len(self.m_h)
        self.ld_h = np.maximum(1, self.m_h) if ld is None else np.asarray(ld, dtype=np.int64)
        self.device = torch.device(device)
        self.offsets, total = _offsets(2 * self.ld_h * self.n_h)    # in doubles
        self.total = total
        self.data = torch.empty(total, dtype=torch.float64, device=self.device)
        self.ptr = torch.from_numpy(self.data.data_ptr() + 8 * self.offsets).to(self.device)
        self.m = torch.from_numpy(self.m_h.astype(np.int32)).to(self.device)
        self.n = torch.from_numpy(self.n_h.astype(np.int32)).to(self.device)
        self.ld = torch.from_numpy(self.ld_h.astype(np.int32)).to(self.device)
        self.max_m = int(self.m_h.max()) if self.batch else 0
        self.max_n = int(self.n_h.max()) if self.batch else 0
        self.k_h = np.minimum(self.m_h, self.n_h)
        self.ipiv_off, ipiv_total = _offsets(self.k_h)
        self.ipiv_data = torch.zeros(ipiv_total, dtype=torch.int32, device=self.device)
        self.ipiv = torch.from_numpy(self.ipiv_data.data_ptr() + 4 * self.ipiv_off).to(self.device)
        self.info = torch.zeros(max(1, self.batch), dtype=torch.int32, device=self.device)
        self.work = None

    def matrix(self, i, flat_host: np.ndarray):
        """complex128 view of matrix i inside a flat float64 host copy of data."""
        o, m, n, ld = int(self.offsets[i]), int(self.m_h[i]), int(self.n_h[i]), int(self.ld_h[i])
        if m * n == 0:
            return np.zeros((m, n), dtype=np.complex128, order="F")
        z = flat_host[o: o + 2 * ld * n].view(np.complex128)
        return np.lib.stride_tricks.as_strided(z, shape=(m, n), strides=(16, 16 * ld))

    def ipiv_of(self, i, ipiv_host: np.ndarray):
        o, k = int(self.ipiv_off[i]), int(self.k_h[i])
        return ipiv_host[o:o + k]

    def workspace(self):
        if self.work is None:
            nb = irr.irr_zgetrf_workspace_size(self.batch, self.max_m, self.max_n)
            self.work = torch.empty(max(256, nb), dtype=torch.uint8, device=self.device)
        return self.work

    def getrf(self, stream=None, max_m=None, max_n=None):
        """irr_zgetrf on the whole batch (asynchronous on `stream`)."""
        return irr.irr_zgetrf(self.batch, self.max_m if max_m is None else max_m,
                              self.max_n if max_n is None else max_n, self.m, self.n, self.ptr, self.ld,
                              self.ipiv, self.info, self.workspace(), stream)

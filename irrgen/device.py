"""Device-side value generator (input construction only, no method arithmetic).

`fill_device` writes the same values as `irrgen.fill_packed` straight into a
device buffer with a small CUDA kernel (irrgen/csrc/irrgen_dev.cu ->
irrgen/libirrgen.so), for batches too large to build on the host (C5: 68 GB).
Byte equality with the host generator is asserted by tests/test_gpu_getrf.py.
"""
from __future__ import annotations

import ctypes as C
import os
import subprocess

import numpy as np

HERE = os.path.dirname(os.path.abspath(__file__))
SRC = os.path.join(HERE, "csrc", "irrgen_dev.cu")
SO = os.path.join(HERE, "libirrgen.so")
NVCC = os.environ.get("NVCC", "/usr/local/cuda/bin/nvcc")

_lib = None


def build(force: bool = False) -> str:
    if force or not os.path.exists(SO) or os.path.getmtime(SO) < os.path.getmtime(SRC):
        tmp = SO + f".tmp{os.getpid()}"
        cmd = [NVCC, "-gencode", "arch=compute_100a,code=sm_100a", "-O3", "-lineinfo", "-std=c++17",
               "-Xcompiler", "-fPIC", "-shared", "-cudart", "static", SRC, "-o", tmp]
        r = subprocess.run(cmd, capture_output=True, text=True)
        if r.returncode != 0:
            raise RuntimeError(f"nvcc failed for {SRC}:\n{r.stdout}\n{r.stderr}")
        os.replace(tmp, SO)
    return SO


def _load():
    global _lib
    if _lib is None:
        if not os.path.exists(SO):
            build()
        L = C.CDLL(SO)
        L.irrgen_fill_device.argtypes = [C.c_int, C.c_void_p, C.c_void_p, C.c_void_p, C.c_void_p, C.c_void_p,
                                         C.c_ulonglong, C.c_void_p, C.c_void_p]
        L.irrgen_fill_device.restype = C.c_int
        _lib = L
    return _lib


class Filler:
    """Device index arrays built once; `fill(out)` regenerates the batch
    (bench.py restores C5 inputs this way between steps, untimed)."""

    def __init__(self, seed: int, m, n, ld, offsets, gids, device):
        import torch
        t32 = lambda a: torch.from_numpy(np.ascontiguousarray(a, dtype=np.int32)).to(device)  # noqa: E731
        t64 = lambda a: torch.from_numpy(np.ascontiguousarray(a, dtype=np.int64)).to(device)  # noqa: E731
        self.count = len(m)
        self.seed = seed
        self.t = (t32(m), t32(n), t32(ld), t64(offsets), t64(gids))

    def fill(self, out, stream=None):
        import torch
        if self.count == 0:
            return out
        s = stream if stream is not None else torch.cuda.current_stream(out.device)
        dm, dn, dl, do, dg = self.t
        rc = _load().irrgen_fill_device(self.count, dm.data_ptr(), dn.data_ptr(), dl.data_ptr(), do.data_ptr(),
                                        dg.data_ptr(), C.c_ulonglong(self.seed & 0xFFFFFFFFFFFFFFFF),
                                        out.data_ptr(), C.c_void_p(s.cuda_stream))
        if rc != 0:
            raise RuntimeError(f"irrgen_fill_device: CUDA error {rc}")
        return out


def fill_device(seed: int, m, n, ld, offsets, out, gids, stream=None):
    """out (a float64 CUDA tensor): matrix g gets uniform_values(seed, gids[g],
    m[g], n[g]) at out[offsets[g] + i + j*ld[g]].  m/n/ld/offsets/gids are host
    arrays; asynchronous on `stream` (default: torch's current stream)."""
    import torch
    dev = out.device
    cnt = len(m)
    if cnt == 0:
        return out
    t32 = lambda a: torch.from_numpy(np.ascontiguousarray(a, dtype=np.int32)).to(dev)  # noqa: E731
    t64 = lambda a: torch.from_numpy(np.ascontiguousarray(a, dtype=np.int64)).to(dev)  # noqa: E731
    dm, dn, dl, do, dg = t32(m), t32(n), t32(ld), t64(offsets), t64(gids)
    s = stream if stream is not None else torch.cuda.current_stream(dev)
    rc = _load().irrgen_fill_device(cnt, dm.data_ptr(), dn.data_ptr(), dl.data_ptr(), do.data_ptr(),
                                    dg.data_ptr(), C.c_ulonglong(seed & 0xFFFFFFFFFFFFFFFF), out.data_ptr(),
                                    C.c_void_p(s.cuda_stream))
    if rc != 0:
        raise RuntimeError(f"irrgen_fill_device: CUDA error {rc}")
    # keep the index arrays alive until the kernel has consumed them
    s.synchronize()
    return out

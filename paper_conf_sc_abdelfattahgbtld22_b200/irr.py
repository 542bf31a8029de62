"""Thin Python binding of libirr.so (include/irr.h): argument marshalling only.

Every step of the computation runs in the CUDA kernels behind the C ABI; this
module only converts torch device tensors to raw pointers.  There is no CPU
fallback: if libirr.so is missing or the device is not a B200 the calls raise.

Tensor conventions (all on the same CUDA device):
    size / leading-dimension / info arrays : torch.int32, shape [batch]
    pointer arrays (A, ipiv, F11, ...)     : torch.int64 holding device addresses
    workspace                              : any tensor with >= *_workspace_size bytes
"""
from __future__ import annotations

import ctypes as C
import os

_PKG = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.path.join(_PKG, "libirr.so")

IRR_NO_TRANS, IRR_TRANS = 0, 1
IRR_LEFT, IRR_RIGHT = 0, 1
IRR_LOWER, IRR_UPPER = 0, 1
IRR_NON_UNIT, IRR_UNIT = 0, 1
IRR_SUCCESS, IRR_ERR_CUDA, IRR_ERR_WORKSPACE, IRR_ERR_UNSUPPORTED, IRR_ERR_DEVICE = 0, 1, 2, 3, 4

EXPORTED = (
    "irr_getrf_workspace_size", "irr_getrf", "irr_getrf_partial_workspace_size", "irr_getrf_partial",
    "irr_gemm_workspace_size", "irr_gemm", "irr_trsm_workspace_size", "irr_trsm", "irr_laswp",
    "irr_getrf_partial_lapack_workspace_size", "irr_getrf_partial_lapack", "irr_zgetrf_workspace_size", "irr_zgetrf",
    "irr_shard_lpt", "irr_shard_lpt_work",
    "irr_getrs_workspace_size", "irr_getrs", "irr_status_words", "irr_extend_add",
    "irr_set_tuning", "irr_get_tuning", "irr_reset_tuning", "irr_launch_count", "irr_version",
    "irr_profile_enable", "irr_profile_collect", "irr_profile_num_classes", "irr_profile_class_name",
    "irr_profile_busy",
)

_lib = None


class IrrError(RuntimeError):
    pass


def load(path: str | None = None):
    """Load libirr.so (built in-tree by paper_conf_sc_abdelfattahgbtld22_b200.build)."""
    global _lib
    if _lib is not None:
        return _lib
    p = path or LIB_PATH
    if not os.path.exists(p):
        raise IrrError(f"libirr.so not found at {p}: run `python -m paper_conf_sc_abdelfattahgbtld22_b200.build` "
                       "(there is no CPU fallback)")
    L = C.CDLL(p)
    vp, i, d, sz = C.c_void_p, C.c_int, C.c_double, C.c_size_t
    L.irr_getrf_workspace_size.argtypes = [i, i, i]
    L.irr_getrf_workspace_size.restype = sz
    L.irr_getrf.argtypes = [i, i, i, vp, vp, vp, vp, vp, vp, vp, sz, vp]
    L.irr_getrf.restype = i
    L.irr_getrf_partial_workspace_size.argtypes = [i, i, i]
    L.irr_getrf_partial_workspace_size.restype = sz
    L.irr_getrf_partial.argtypes = [i, i, i, vp, vp, vp, vp, vp, vp, vp, vp, vp, vp, vp, vp, vp, sz, vp]
    L.irr_getrf_partial.restype = i
    L.irr_getrf_partial_lapack_workspace_size.argtypes = [i, i, i]
    L.irr_getrf_partial_lapack_workspace_size.restype = sz
    L.irr_getrf_partial_lapack.argtypes = [i, i, i, vp, vp, vp, vp, vp, vp, vp, vp, vp, vp, vp, vp, vp, sz, vp]
    L.irr_getrf_partial_lapack.restype = i
    L.irr_zgetrf_workspace_size.argtypes = [i, i, i]
    L.irr_zgetrf_workspace_size.restype = sz
    L.irr_zgetrf.argtypes = [i, i, i, vp, vp, vp, vp, vp, vp, vp, sz, vp]
    L.irr_zgetrf.restype = i
    L.irr_shard_lpt.argtypes = [i, vp, vp, i, vp]
    L.irr_shard_lpt.restype = i
    L.irr_shard_lpt_work.argtypes = [i, vp, i, vp]
    L.irr_shard_lpt_work.restype = i
    L.irr_gemm_workspace_size.argtypes = [i]
    L.irr_gemm_workspace_size.restype = sz
    L.irr_gemm.argtypes = [i, i, i, i, i, vp, vp, vp, d, vp, i, i, vp, vp, i, i, vp, d, vp, i, i, vp, i, vp, sz, vp]
    L.irr_gemm.restype = i
    L.irr_trsm_workspace_size.argtypes = [i]
    L.irr_trsm_workspace_size.restype = sz
    L.irr_trsm.argtypes = [i, i, i, i, i, i, vp, vp, d, vp, i, i, vp, vp, i, i, vp, i, vp, sz, vp]
    L.irr_trsm.restype = i
    L.irr_laswp.argtypes = [i, vp, vp, i, i, vp, i, i, vp, vp, i, vp]
    L.irr_laswp.restype = i
    L.irr_getrs_workspace_size.argtypes = [i]
    L.irr_getrs_workspace_size.restype = sz
    L.irr_getrs.argtypes = [i, i, i, i, vp, vp, vp, vp, vp, vp, vp, vp, vp, sz, vp]
    L.irr_getrs.restype = i
    L.irr_extend_add.argtypes = [i, i, vp, vp, vp, vp, vp, vp, vp, vp, vp]
    L.irr_extend_add.restype = i
    L.irr_status_words.argtypes = [i, vp, vp, vp, vp, vp, vp]
    L.irr_status_words.restype = i
    L.irr_set_tuning.argtypes = [C.c_char_p, i]
    L.irr_set_tuning.restype = None
    L.irr_get_tuning.argtypes = [C.c_char_p]
    L.irr_get_tuning.restype = i
    L.irr_reset_tuning.argtypes = []
    L.irr_reset_tuning.restype = None
    L.irr_launch_count.argtypes = [i]
    L.irr_launch_count.restype = C.c_longlong
    L.irr_version.restype = C.c_char_p
    L.irr_profile_enable.argtypes = [i]
    L.irr_profile_enable.restype = i
    L.irr_profile_collect.argtypes = [C.POINTER(C.c_double), C.POINTER(C.c_longlong), i]
    L.irr_profile_collect.restype = i
    L.irr_profile_num_classes.restype = i
    L.irr_profile_busy.argtypes = [C.POINTER(C.c_double), i]
    L.irr_profile_busy.restype = i
    L.irr_profile_class_name.argtypes = [i]
    L.irr_profile_class_name.restype = C.c_char_p
    _lib = L
    return L


def _p(t):
    """Device pointer of a tensor (or None -> NULL)."""
    if t is None:
        return None
    if isinstance(t, int):
        return t
    return t.data_ptr()


def _nbytes(t):
    return 0 if t is None else t.numel() * t.element_size()


def _stream(stream):
    if stream is None:
        import torch
        return torch.cuda.current_stream().cuda_stream
    if isinstance(stream, int):
        return stream
    return stream.cuda_stream


def _check(rc: int, name: str):
    if rc != 0:
        raise IrrError(f"{name} returned {rc}")
    return rc


# ---------------------------------------------------------------- entry points
def irr_getrf_workspace_size(batch, max_m, max_n):
    return load().irr_getrf_workspace_size(batch, max_m, max_n)


def irr_getrf(batch, max_m, max_n, m, n, A, ld, ipiv, info, work, stream=None, check=True):
    rc = load().irr_getrf(batch, max_m, max_n, _p(m), _p(n), _p(A), _p(ld), _p(ipiv), _p(info), _p(work),
                          _nbytes(work), _stream(stream))
    return _check(rc, "irr_getrf") if check else rc


def irr_getrf_partial_workspace_size(batch, max_n1, max_n2):
    return load().irr_getrf_partial_workspace_size(batch, max_n1, max_n2)


def irr_getrf_partial(batch, max_n1, max_n2, n1, n2, F11, ld11, F12, ld12, F21, ld21, F22, ld22, ipiv, info,
                      work, stream=None, check=True):
    rc = load().irr_getrf_partial(batch, max_n1, max_n2, _p(n1), _p(n2), _p(F11), _p(ld11), _p(F12), _p(ld12),
                                  _p(F21), _p(ld21), _p(F22), _p(ld22), _p(ipiv), _p(info), _p(work),
                                  _nbytes(work), _stream(stream))
    return _check(rc, "irr_getrf_partial") if check else rc


def irr_getrf_partial_lapack_workspace_size(batch, max_n1, max_n2):
    return load().irr_getrf_partial_lapack_workspace_size(batch, max_n1, max_n2)


def irr_getrf_partial_lapack(batch, max_n1, max_n2, n1, n2, F11, ld11, F12, ld12, F21, ld21, F22, ld22, ipiv,
                             info, work, stream=None, check=True):
    rc = load().irr_getrf_partial_lapack(batch, max_n1, max_n2, _p(n1), _p(n2), _p(F11), _p(ld11), _p(F12),
                                         _p(ld12), _p(F21), _p(ld21), _p(F22), _p(ld22), _p(ipiv), _p(info),
                                         _p(work), _nbytes(work), _stream(stream))
    return _check(rc, "irr_getrf_partial_lapack") if check else rc


def irr_zgetrf_workspace_size(batch, max_m, max_n):
    return load().irr_zgetrf_workspace_size(batch, max_m, max_n)


def irr_zgetrf(batch, max_m, max_n, m, n, A, ld, ipiv, info, work, stream=None, check=True):
    rc = load().irr_zgetrf(batch, max_m, max_n, _p(m), _p(n), _p(A), _p(ld), _p(ipiv), _p(info), _p(work),
                           _nbytes(work), _stream(stream))
    return _check(rc, "irr_zgetrf") if check else rc


def irr_shard_lpt_work(work, parts: int):
    """Host LPT partition through the C ABI: owner (int32 numpy array)."""
    import numpy as np
    w = np.ascontiguousarray(work, dtype=np.float64)
    owner = np.zeros(max(1, len(w)), dtype=np.int32)
    rc = load().irr_shard_lpt_work(len(w), w.ctypes.data, int(parts), owner.ctypes.data)
    _check(rc, "irr_shard_lpt_work")
    return owner[: len(w)]


def irr_getrs_workspace_size(batch):
    return load().irr_getrs_workspace_size(batch)


def irr_getrs(trans, batch, max_n, max_nrhs, n, nrhs, A, lda, ipiv, B, ldb, info, work, stream=None, check=True):
    rc = load().irr_getrs(trans, batch, max_n, max_nrhs, _p(n), _p(nrhs), _p(A), _p(lda), _p(ipiv), _p(B),
                          _p(ldb), _p(info), _p(work), _nbytes(work), _stream(stream))
    return _check(rc, "irr_getrs") if check else rc


def irr_extend_add(batch, max_n2, n2, F22, ld22, rel, np_, Fp, ldp, info, stream=None, check=True):
    rc = load().irr_extend_add(batch, max_n2, _p(n2), _p(F22), _p(ld22), _p(rel), _p(np_), _p(Fp), _p(ldp),
                               _p(info), _stream(stream))
    return _check(rc, "irr_extend_add") if check else rc


def irr_status_words(batch, m, n, ipiv, info, words, stream=None, check=True):
    rc = load().irr_status_words(batch, _p(m), _p(n), _p(ipiv), _p(info), _p(words), _stream(stream))
    return _check(rc, "irr_status_words") if check else rc


def irr_gemm_workspace_size(batch):
    return load().irr_gemm_workspace_size(batch)


def irr_gemm(ta, tb, max_m, max_n, max_k, m, n, k, alpha, A, Ai, Aj, lda, B, Bi, Bj, ldb, beta, Cp, Ci, Cj, ldc,
             batch, work=None, stream=None, check=True):
    rc = load().irr_gemm(ta, tb, max_m, max_n, max_k, _p(m), _p(n), _p(k), float(alpha), _p(A), Ai, Aj, _p(lda),
                         _p(B), Bi, Bj, _p(ldb), float(beta), _p(Cp), Ci, Cj, _p(ldc), batch, _p(work),
                         _nbytes(work), _stream(stream))
    return _check(rc, "irr_gemm") if check else rc


def irr_trsm_workspace_size(batch):
    return load().irr_trsm_workspace_size(batch)


def irr_trsm(side, uplo, trans, diag, max_m, max_n, m, n, alpha, T, Ti, Tj, ldt, B, Bi, Bj, ldb, batch,
             work=None, stream=None, check=True):
    rc = load().irr_trsm(side, uplo, trans, diag, max_m, max_n, _p(m), _p(n), float(alpha), _p(T), Ti, Tj,
                         _p(ldt), _p(B), Bi, Bj, _p(ldb), batch, _p(work), _nbytes(work), _stream(stream))
    return _check(rc, "irr_trsm") if check else rc


def irr_laswp(max_n, n, A, Ai, Aj, lda, k1, k2, kcount, ipiv, batch, stream=None, check=True):
    rc = load().irr_laswp(max_n, _p(n), _p(A), Ai, Aj, _p(lda), k1, k2, _p(kcount), _p(ipiv), batch,
                          _stream(stream))
    return _check(rc, "irr_laswp") if check else rc


def irr_set_tuning(key: str, value: int):
    load().irr_set_tuning(key.encode(), int(value))


def irr_get_tuning(key: str) -> int:
    return load().irr_get_tuning(key.encode())


def irr_reset_tuning():
    load().irr_reset_tuning()


def irr_launch_count(reset: bool = False) -> int:
    return load().irr_launch_count(1 if reset else 0)


def irr_version() -> str:
    return load().irr_version().decode()


def irr_profile_enable(max_launches: int):
    return _check(load().irr_profile_enable(int(max_launches)), "irr_profile_enable")


def irr_profile_busy():
    """{class name: ms} -- per class the union of its launch intervals since the
    last collect (overlapping launches on several streams counted once); call
    before irr_profile_collect."""
    L = load()
    nc = L.irr_profile_num_classes()
    ms = (C.c_double * nc)()
    if L.irr_profile_busy(ms, nc) < 0:
        raise IrrError("irr_profile_busy failed")
    return {L.irr_profile_class_name(c).decode(): ms[c] for c in range(nc)}


def irr_profile_collect():
    """{class name: (ms, launches)} since the last collect (waits for the events)."""
    L = load()
    nc = L.irr_profile_num_classes()
    ms = (C.c_double * nc)()
    cnt = (C.c_longlong * nc)()
    if L.irr_profile_collect(ms, cnt, nc) < 0:
        raise IrrError("irr_profile_collect failed")
    return {L.irr_profile_class_name(c).decode(): (ms[c], cnt[c]) for c in range(nc)}

"""ctypes front-end of the plain CPU oracle (oracle/oracle.c).

TEST INFRASTRUCTURE ONLY: imported by tests/, __graft_entry__.smoke() and the
cpu_baseline / --impl reference legs of bench.py -- never by the product
package.  The oracle shares no code with the CUDA path.

Every function here only marshals numpy arrays into the C oracle; the
arithmetic is in oracle.c (see its header for the PAPER.md citations).
Matrices are numpy arrays in Fortran (column-major) order.
"""
from __future__ import annotations

import ctypes as C
import os
import subprocess

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SO = os.path.join(_HERE, "liboracle.so")
_SRC = os.path.join(_HERE, "oracle.c")
_CHECK = os.path.join(_HERE, "check.c")   # batched parity checker (calls the oracle; no method arithmetic)
_lib = None

CFLAGS = ["-O2", "-ffp-contract=off", "-fno-fast-math", "-fopenmp", "-shared", "-fPIC", "-std=c11"]


def build(force: bool = False) -> str:
    """Compile oracle.c -> liboracle.so (gcc, no FMA contraction, no fast-math)."""
    newest = max(os.path.getmtime(_SRC), os.path.getmtime(_CHECK))
    if force or not os.path.exists(_SO) or os.path.getmtime(_SO) < newest:
        tmp = _SO + f".tmp{os.getpid()}"
        subprocess.check_call(["gcc", *CFLAGS, "-o", tmp, _SRC, _CHECK, "-lm"])
        os.replace(tmp, _SO)
    return _SO


def lib():
    global _lib
    if _lib is None:
        build()
        L = C.CDLL(_SO)
        P = C.POINTER
        dp, ip = P(C.c_double), P(C.c_int)
        L.oracle_getrf.argtypes = [C.c_int, C.c_int, dp, C.c_int, ip, ip, dp]
        L.oracle_getrf_batch.argtypes = [C.c_int, ip, ip, P(dp), ip, P(ip), ip, dp, C.c_int]
        L.oracle_getrf_partial.argtypes = [C.c_int, C.c_int, dp, C.c_int, dp, C.c_int, dp, C.c_int,
                                           dp, C.c_int, ip, ip]
        L.oracle_getrf_partial_batch.argtypes = [C.c_int, ip, ip, P(dp), ip, P(dp), ip, P(dp), ip,
                                                 P(dp), ip, P(ip), ip, C.c_int]
        L.oracle_gemm.argtypes = [C.c_int, C.c_int, C.c_int, C.c_int, C.c_int, C.c_double, dp, C.c_int,
                                  dp, C.c_int, C.c_double, dp, C.c_int]
        L.oracle_trsm.argtypes = [C.c_int] * 6 + [C.c_double, dp, C.c_int, dp, C.c_int]
        L.oracle_laswp.argtypes = [C.c_int, dp, C.c_int, C.c_int, C.c_int, ip]
        L.oracle_getrs.argtypes = [C.c_int, C.c_int, dp, C.c_int, ip, dp, C.c_int]
        L.oracle_getrs.restype = C.c_int
        L.oracle_extend_add.argtypes = [C.c_int, dp, C.c_int, ip, C.c_int, dp, C.c_int]
        L.oracle_extend_add.restype = C.c_int
        L.oracle_backward_error.argtypes = [C.c_int, C.c_int, dp, C.c_int, dp, C.c_int, ip]
        L.oracle_backward_error.restype = C.c_double
        L.oracle_num_threads.restype = C.c_int
        L.oracle_getrf_partial_lapack.argtypes = [C.c_int, C.c_int, dp, C.c_int, dp, C.c_int, dp, C.c_int,
                                                  dp, C.c_int, ip, ip]
        L.oracle_zgetrf.argtypes = [C.c_int, C.c_int, dp, C.c_int, ip, ip, dp]
        L.oracle_zbackward_error.argtypes = [C.c_int, C.c_int, dp, C.c_int, dp, C.c_int, ip]
        L.oracle_zbackward_error.restype = C.c_double
        vp = C.c_void_p
        L.check_getrf_batch.argtypes = [C.c_int, vp, vp, vp, vp, vp, vp, vp, vp, vp, C.c_int]
        L.check_getrf_batch.restype = C.c_int
        L.check_partial_batch.argtypes = [C.c_int, vp, vp, vp, vp, vp, vp, vp, vp, vp, C.c_int]
        L.check_partial_batch.restype = C.c_int
        _lib = L
    return _lib


def _dp(a):
    return a.ctypes.data_as(C.POINTER(C.c_double))


def _ip(a):
    return a.ctypes.data_as(C.POINTER(C.c_int))


def _fortran(A):
    A = np.asarray(A, dtype=np.float64)
    if A.ndim != 2:
        raise ValueError("matrix must be 2-D")
    return np.array(A, dtype=np.float64, order="F", copy=True)


def _ld(A):
    return max(1, A.shape[0]) if A.size == 0 else A.strides[1] // 8


def getrf(A):
    """GEPP on a copy of A.  Returns (LU, ipiv (1-based int32), info, min_sep)."""
    LU = _fortran(A)
    m, n = LU.shape
    ipiv = np.zeros(max(1, min(m, n)), dtype=np.int32)
    info = np.zeros(1, dtype=np.int32)
    sep = np.zeros(1)
    buf = LU if LU.size else np.zeros((max(1, m), 1), order="F")
    r = lib().oracle_getrf(m, n, _dp(buf), max(1, m), _ip(ipiv), _ip(info), _dp(sep))
    if r < 0:
        raise ValueError(f"oracle_getrf: bad argument {-r}")
    return LU, ipiv[: min(m, n)], int(info[0]), float(sep[0])


def getrf_batch(mats, nthreads: int = 0):
    """Batched GEPP in place on a list of Fortran float64 arrays (OpenMP over
    matrices).  Returns (ipivs, info, min_sep)."""
    b = len(mats)
    m = np.array([M.shape[0] for M in mats], dtype=np.int32)
    n = np.array([M.shape[1] for M in mats], dtype=np.int32)
    ld = np.array([max(1, M.shape[0]) for M in mats], dtype=np.int32)
    keep = []
    ptrs = (C.POINTER(C.c_double) * max(1, b))()
    ipivs = [np.zeros(max(1, min(M.shape)), dtype=np.int32) for M in mats]
    iptrs = (C.POINTER(C.c_int) * max(1, b))()
    for i, M in enumerate(mats):
        if not (M.flags.f_contiguous and M.dtype == np.float64):
            raise ValueError("matrices must be Fortran float64")
        buf = M if M.size else np.zeros(1)
        keep.append(buf)
        ptrs[i] = _dp(buf)
        iptrs[i] = _ip(ipivs[i])
    info = np.zeros(max(1, b), dtype=np.int32)
    sep = np.zeros(max(1, b))
    lib().oracle_getrf_batch(b, _ip(m), _ip(n), ptrs, _ip(ld), iptrs, _ip(info), _dp(sep), nthreads)
    return [p[: min(M.shape)] for p, M in zip(ipivs, mats)], info[:b], sep[:b]


def getrf_partial(F11, F12, F21, F22):
    """Partial front factorization on copies.
    Returns (F11 -> L\\U, F12 -> U^-1 L^-1 P^T F12, F22 -> F22 - F21 F12, ipiv, info)."""
    F11, F12, F21, F22 = (_fortran(X) for X in (F11, F12, F21, F22))
    n1, n2 = F11.shape[0], F22.shape[0]
    ipiv = np.zeros(max(1, n1), dtype=np.int32)
    info = np.zeros(1, dtype=np.int32)
    bufs = [X if X.size else np.zeros(1) for X in (F11, F12, F21, F22)]
    r = lib().oracle_getrf_partial(n1, n2, _dp(bufs[0]), max(1, n1), _dp(bufs[1]), max(1, n1),
                                   _dp(bufs[2]), max(1, n2), _dp(bufs[3]), max(1, n2), _ip(ipiv), _ip(info))
    if r < 0:
        raise ValueError(f"oracle_getrf_partial: bad argument {-r}")
    return F11, F12, F22, ipiv[:n1], int(info[0])


def getrf_partial_lapack(F11, F12, F21, F22):
    """LAPACK-style partial front on copies.  Returns
    (F11 -> L\\U, F12 -> U12 = L^-1 P^T F12, F21 -> L21 = F21 U^-1,
    F22 -> F22 - L21 U12, ipiv, info)."""
    F11, F12, F21, F22 = (_fortran(X) for X in (F11, F12, F21, F22))
    n1, n2 = F11.shape[0], F22.shape[0]
    ipiv = np.zeros(max(1, n1), dtype=np.int32)
    info = np.zeros(1, dtype=np.int32)
    bufs = [X if X.size else np.zeros(1) for X in (F11, F12, F21, F22)]
    r = lib().oracle_getrf_partial_lapack(n1, n2, _dp(bufs[0]), max(1, n1), _dp(bufs[1]), max(1, n1),
                                          _dp(bufs[2]), max(1, n2), _dp(bufs[3]), max(1, n2), _ip(ipiv),
                                          _ip(info))
    if r < 0:
        raise ValueError(f"oracle_getrf_partial_lapack: bad argument {-r}")
    return F11, F12, F21, F22, ipiv[:n1], int(info[0])


def _cfortran(A):
    A = np.asarray(A, dtype=np.complex128)
    if A.ndim != 2:
        raise ValueError("matrix must be 2-D")
    return np.array(A, dtype=np.complex128, order="F", copy=True)


def zgetrf(A):
    """Complex GEPP (LAPACK zgetf2 semantics, izamax pivoting) on a copy of A.
    Returns (LU complex128 Fortran, ipiv (1-based int32), info, min_sep)."""
    LU = _cfortran(A)
    m, n = LU.shape
    ipiv = np.zeros(max(1, min(m, n)), dtype=np.int32)
    info = np.zeros(1, dtype=np.int32)
    sep = np.zeros(1)
    buf = LU if LU.size else np.zeros((max(1, m), 1), dtype=np.complex128, order="F")
    r = lib().oracle_zgetrf(m, n, buf.ctypes.data_as(C.POINTER(C.c_double)), max(1, m), _ip(ipiv), _ip(info),
                            _dp(sep))
    if r < 0:
        raise ValueError(f"oracle_zgetrf: bad argument {-r}")
    return LU, ipiv[: min(m, n)], int(info[0]), float(sep[0])


def zbackward_error(A0, LU, ipiv):
    A0, LU = _cfortran(A0), _cfortran(LU)
    m, n = A0.shape
    ipiv = np.ascontiguousarray(ipiv, dtype=np.int32)
    if ipiv.size == 0:
        ipiv = np.zeros(1, dtype=np.int32)
    z = np.zeros((1, 1), dtype=np.complex128, order="F")
    b0 = A0 if A0.size else z
    b1 = LU if LU.size else z
    P = C.POINTER(C.c_double)
    return lib().oracle_zbackward_error(m, n, b0.ctypes.data_as(P), max(1, m), b1.ctypes.data_as(P), max(1, m),
                                        _ip(ipiv))


def getrf_partial_batch(fronts, nthreads: int = 0):
    """fronts: list of dicts with Fortran arrays F11, F12, F21, F22 (modified
    in place).  Returns (ipivs, info)."""
    b = len(fronts)
    n1 = np.array([f["F11"].shape[0] for f in fronts], dtype=np.int32)
    n2 = np.array([f["F22"].shape[0] for f in fronts], dtype=np.int32)
    P = C.POINTER(C.c_double)
    arrs = {k: (P * max(1, b))() for k in ("F11", "F12", "F21", "F22")}
    lds = {k: np.zeros(max(1, b), dtype=np.int32) for k in arrs}
    keep = []
    ipivs = [np.zeros(max(1, int(x)), dtype=np.int32) for x in n1]
    iptrs = (C.POINTER(C.c_int) * max(1, b))()
    for i, f in enumerate(fronts):
        for k in arrs:
            X = f[k]
            if X.size and not (X.dtype == np.float64 and X.strides[0] == 8):
                raise ValueError("fronts must be column-major float64")
            buf = X if X.size else np.zeros(1)
            keep.append(buf)
            arrs[k][i] = _dp(buf)
            lds[k][i] = max(1, X.strides[1] // 8 if X.size else X.shape[0])
        iptrs[i] = _ip(ipivs[i])
    info = np.zeros(max(1, b), dtype=np.int32)
    lib().oracle_getrf_partial_batch(b, _ip(n1), _ip(n2), arrs["F11"], _ip(lds["F11"]), arrs["F12"],
                                     _ip(lds["F12"]), arrs["F21"], _ip(lds["F21"]), arrs["F22"],
                                     _ip(lds["F22"]), iptrs, _ip(info), nthreads)
    return [p[: int(k)] for p, k in zip(ipivs, n1)], info[:b]


def gemm(ta, tb, alpha, A, B, beta, C_):
    A, B, Cm = _fortran(A), _fortran(B), _fortran(C_)
    m, n = Cm.shape
    k = A.shape[0] if ta else A.shape[1]
    bufs = [X if X.size else np.zeros((1, 1), order="F") for X in (A, B, Cm)]
    lib().oracle_gemm(int(ta), int(tb), m, n, k, float(alpha), _dp(bufs[0]), max(1, A.shape[0]),
                      _dp(bufs[1]), max(1, B.shape[0]), float(beta), _dp(bufs[2]), max(1, m))
    return Cm


def trsm(side, uplo, trans, diag, alpha, T, B):
    T, B = _fortran(T), _fortran(B)
    m, n = B.shape
    bufs = [X if X.size else np.zeros((1, 1), order="F") for X in (T, B)]
    lib().oracle_trsm(int(side), int(uplo), int(trans), int(diag), m, n, float(alpha),
                      _dp(bufs[0]), max(1, T.shape[0]), _dp(bufs[1]), max(1, m))
    return B


def laswp(A, k1, k2, ipiv):
    A = _fortran(A)
    ipiv = np.ascontiguousarray(ipiv, dtype=np.int32)
    buf = A if A.size else np.zeros((1, 1), order="F")
    lib().oracle_laswp(A.shape[1], _dp(buf), max(1, A.shape[0]), int(k1), int(k2), _ip(ipiv))
    return A


def getrs(LU, ipiv, B):
    """X = A^-1 B from the factors of getrf (LU n x n, 1-based ipiv), on a copy of B."""
    LU, B = _fortran(LU), _fortran(B)
    n = LU.shape[0]
    nrhs = B.shape[1]
    ipiv = np.ascontiguousarray(ipiv, dtype=np.int32)
    if ipiv.size == 0:
        ipiv = np.zeros(1, dtype=np.int32)
    b0 = LU if LU.size else np.zeros((1, 1), order="F")
    b1 = B if B.size else np.zeros((1, 1), order="F")
    r = lib().oracle_getrs(n, nrhs, _dp(b0), max(1, n), _ip(ipiv), _dp(b1), max(1, n))
    if r < 0:
        raise ValueError(f"oracle_getrs: bad argument {-r}")
    return B


def extend_add(Fp, F22, rel):
    """Fp[rel_i, rel_j] += F22[i, j], on a copy of the np x np parent front Fp."""
    Fp, F22 = _fortran(Fp), _fortran(F22)
    n2, npp = F22.shape[0], Fp.shape[0]
    rel = np.ascontiguousarray(rel, dtype=np.int32)
    r0 = rel if rel.size else np.zeros(1, dtype=np.int32)
    b0 = F22 if F22.size else np.zeros((1, 1), order="F")
    b1 = Fp if Fp.size else np.zeros((1, 1), order="F")
    r = lib().oracle_extend_add(n2, _dp(b0), max(1, n2), _ip(r0), npp, _dp(b1), max(1, npp))
    if r < 0:
        raise ValueError(f"oracle_extend_add: bad argument {-r}")
    return Fp


def backward_error(A0, LU, ipiv):
    A0, LU = _fortran(A0), _fortran(LU)
    m, n = A0.shape
    ipiv = np.ascontiguousarray(ipiv, dtype=np.int32)
    if ipiv.size == 0:
        ipiv = np.zeros(1, dtype=np.int32)
    b0 = A0 if A0.size else np.zeros((1, 1), order="F")
    b1 = LU if LU.size else np.zeros((1, 1), order="F")
    return lib().oracle_backward_error(m, n, _dp(b0), max(1, m), _dp(b1), max(1, m), _ip(ipiv))


def num_threads() -> int:
    return lib().oracle_num_threads()


# ---------------------------------------------------------------------------
# Batched parity records (check.c): every matrix of a packed batch against the
# oracle, without a Python object per matrix.  Field names of one record:
GETRF_FIELDS = ("info_o", "ipiv_eq", "first_diff", "be", "dl", "du", "rho", "lmax", "exact")
PARTIAL_FIELDS = GETRF_FIELDS + ("f21_same", "d12", "d22", "front_exact")


def _ptrs(flat, offsets, itemsize):
    """Device-style pointer array (uint64) into a flat host buffer."""
    base = flat.ctypes.data
    return (np.uint64(base) + np.asarray(offsets, dtype=np.uint64) * np.uint64(itemsize)).astype(np.uint64)


def _i32(x):
    return np.ascontiguousarray(x, dtype=np.int32)


def check_getrf_packed(m, n, A0, ld0, off0, LU, ld, off, ipiv, ipiv_off, info, nthreads: int = 0):
    """Records (batch x len(GETRF_FIELDS)) comparing the GPU results (LU, ipiv,
    info in packed host buffers) with oracle_getrf of the originals A0."""
    m, n, ld0, ld, info = _i32(m), _i32(n), _i32(ld0), _i32(ld), _i32(info)
    b = len(m)
    pa, pl = _ptrs(A0, off0, 8), _ptrs(LU, off, 8)
    pi = _ptrs(ipiv, ipiv_off, 4)
    out = np.empty((max(1, b), len(GETRF_FIELDS)))
    nf = lib().check_getrf_batch(b, m.ctypes.data, n.ctypes.data, pa.ctypes.data, ld0.ctypes.data, pl.ctypes.data,
                                 ld.ctypes.data, pi.ctypes.data, info.ctypes.data, out.ctypes.data, nthreads)
    assert nf == len(GETRF_FIELDS)
    return out[:b]


def check_partial_packed(n1, n2, F0, ld0, off0, Fg, ld, off, ipiv, ipiv_off, info, nthreads: int = 0):
    """Records (batch x len(PARTIAL_FIELDS)) for fronts stored as one nf x nf
    block each (nf = n1 + n2), GPU results against oracle_getrf_partial."""
    n1, n2, ld0, ld, info = _i32(n1), _i32(n2), _i32(ld0), _i32(ld), _i32(info)
    b = len(n1)
    pa, pf = _ptrs(F0, off0, 8), _ptrs(Fg, off, 8)
    pi = _ptrs(ipiv, ipiv_off, 4)
    out = np.empty((max(1, b), len(PARTIAL_FIELDS)))
    nf = lib().check_partial_batch(b, n1.ctypes.data, n2.ctypes.data, pa.ctypes.data, ld0.ctypes.data,
                                   pf.ctypes.data, ld.ctypes.data, pi.ctypes.data, info.ctypes.data,
                                   out.ctypes.data, nthreads)
    assert nf == len(PARTIAL_FIELDS)
    return out[:b]

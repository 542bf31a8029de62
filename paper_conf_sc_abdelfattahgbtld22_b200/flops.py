"""Operation and byte counts used by the metric (host-side bookkeeping only).

FLOPS_DGETRF (SURVEY.md §8(c) reading Q1): the paper prints the LU count as
"M N^2 - N^2/3 - N^2/2 + 5N/6" (§III-B, garbled: the second term
is N^3/3) and the square case with "+ n^2/2" (L201 §V-A, a sign slip against
L106/L186).  We use LAPACK/MAGMA FLOPS_DGETRF:
    m >= n :  m n^2 - n^3/3 - n^2/2 + 5n/6
    m <  n :  n m^2 - m^3/3 - m^2/2 + 5m/6
Partial front (reading Q2): FLOPS_DGETRF(n1, n1) + 2 n1^2 n2 (two TRSMs, each
counted n m^2 as in L182) + 2 n1 n2^2 (the Schur GEMM, L97).

Algorithmic bytes: each matrix read once and written once,
plus its ipiv, sizes, pointers and info:
    getrf : 16 m n + 4 min(m,n) + 32
    front : 8 (2 n1^2 + 2 n1 n2 + n2 n1 + 2 n2^2) + 4 n1 + 64   (F21 read-only)
"""
from __future__ import annotations

import numpy as np


def getrf_flops(m, n):
    m = np.asarray(m, dtype=np.float64)
    n = np.asarray(n, dtype=np.float64)
    big = np.maximum(m, n)
    k = np.minimum(m, n)
    f = big * k * k - k ** 3 / 3.0 - k * k / 2.0 + 5.0 * k / 6.0
    return np.where(k > 0, f, 0.0)


def partial_flops(n1, n2):
    n1 = np.asarray(n1, dtype=np.float64)
    n2 = np.asarray(n2, dtype=np.float64)
    return getrf_flops(n1, n1) + 2.0 * n1 * n1 * n2 + 2.0 * n1 * n2 * n2


def getrf_bytes(m, n):
    m = np.asarray(m, dtype=np.float64)
    n = np.asarray(n, dtype=np.float64)
    return 16.0 * m * n + 4.0 * np.minimum(m, n) + 32.0


def partial_bytes(n1, n2):
    n1 = np.asarray(n1, dtype=np.float64)
    n2 = np.asarray(n2, dtype=np.float64)
    return 8.0 * (2 * n1 * n1 + 2 * n1 * n2 + n2 * n1 + 2 * n2 * n2) + 4.0 * n1 + 64.0

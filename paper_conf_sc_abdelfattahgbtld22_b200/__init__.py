"""B200-native irrLU: variable-size batched LU with partial pivoting (sm_100a).

The product is the C-ABI library libirr.so (include/irr.h, sources in csrc/);
`irr` is its thin ctypes binding and `batch` builds caller-owned device
layouts.  There is no CPU fallback.
"""
from . import flops, irr  # noqa: F401

__all__ = ["flops", "irr"]

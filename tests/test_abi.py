"""The C ABI: the library loads without a GPU and exports every function
declared in include/irr.h (CPU-only)."""
import ctypes
import os
import re

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def declared_functions():
    src = open(os.path.join(ROOT, "include", "irr.h")).read()
    src = re.sub(r"/\*.*?\*/", "", src, flags=re.S)
    return sorted(set(re.findall(r"\b(irr_[a-z_]+)\s*\(", src)))


def test_library_exports_every_declared_symbol():
    from paper_conf_sc_abdelfattahgbtld22_b200 import build, irr
    build.build()
    lib = ctypes.CDLL(irr.LIB_PATH)
    names = declared_functions()
    assert len(names) >= 14
    for name in names:
        assert hasattr(lib, name), name
    assert set(irr.EXPORTED) == set(names)


def test_host_only_entry_points():
    """Queries and tuning need no device; argument errors return -position."""
    from paper_conf_sc_abdelfattahgbtld22_b200 import irr
    L = irr.load()
    assert irr.irr_version().startswith("irrlu-b200")
    assert irr.irr_getrf_workspace_size(1000, 256, 256) >= 1000 * 5 * 4
    assert irr.irr_gemm_workspace_size(10) > 0
    irr.irr_set_tuning("nb", 16)
    assert irr.irr_get_tuning("nb") == 16
    irr.irr_reset_tuning()
    assert irr.irr_get_tuning("nb") == 32
    assert irr.irr_get_tuning("bogus") == -1
    # bad host arguments are rejected before any device work
    assert L.irr_getrf(-1, 1, 1, None, None, None, None, None, None, None, 0, None) == -1
    assert L.irr_getrf(0, 1, 1, None, None, None, None, None, None, None, 0, None) == 0
    assert L.irr_getrf(3, 1, 1, None, None, None, None, None, None, None, 0, None) == -4
    assert L.irr_laswp(-1, None, None, 0, 0, None, 0, 1, None, None, 1, None) == -1
    assert L.irr_trsm(7, 0, 0, 0, 1, 1, None, None, 1.0, None, 0, 0, None, None, 0, 0, None, 1, None, 0, None) == -1


def test_no_cpu_fallback_without_library(tmp_path):
    from paper_conf_sc_abdelfattahgbtld22_b200 import irr
    import pytest
    saved = irr._lib
    try:
        irr._lib = None
        with pytest.raises(irr.IrrError):
            irr.load(str(tmp_path / "missing.so"))
    finally:
        irr._lib = saved

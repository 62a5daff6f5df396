"""CPU-side checks of the boundary: the C-ABI library loads (no GPU needed to
load it) and exports every function include/*.h declares; the binding's struct
layouts match the header's sizes."""
import ctypes
import os
import re

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def declared_functions():
    names = set()
    for h in ("xpl.h",):
        text = open(os.path.join(ROOT, "include", h)).read()
        text = re.sub(r"/\*.*?\*/", "", text, flags=re.S)
        names |= set(re.findall(r"^\s*(?:const\s+)?\w+\*?\s+\*?(xpl_\w+)\s*\(", text, flags=re.M))
    return sorted(names)


def test_header_declares_the_boundary():
    names = declared_functions()
    for f in ("xpl_init", "xpl_finalize", "xpl_register_alloc", "xpl_free", "xpl_kernel_begin",
              "xpl_kernel_end", "xpl_record_host", "xpl_record_copy", "xpl_diagnose",
              "xpl_get_device_ctx", "xpl_status_string"):
        assert f in names


def test_library_exports_every_declared_symbol():
    from paper_conf_ipps_pirkelbauerlvl20_b200 import LIB_PATH, WORK_PATH
    if not os.path.exists(LIB_PATH):
        import __graft_entry__
        __graft_entry__.build()
    lib = ctypes.CDLL(LIB_PATH)
    missing = [n for n in declared_functions() if not hasattr(lib, n)]
    assert not missing, missing
    work = ctypes.CDLL(WORK_PATH)
    assert hasattr(work, "xplw_bind") and hasattr(work, "xplw_replay")


def test_binding_struct_sizes():
    from paper_conf_ipps_pirkelbauerlvl20_b200 import xpl
    assert ctypes.sizeof(xpl.XplAllocReport) == 4 * 8 + 4 * 4 + 18 * 8
    assert xpl.HOST_ACCESS_DTYPE.itemsize == 16
    assert ctypes.sizeof(xpl.XplDiagParams) == 24
    # every function the binding wraps is a declared one
    assert set(xpl.EXPORTED) <= set(declared_functions())


def test_status_string_without_gpu():
    from paper_conf_ipps_pirkelbauerlvl20_b200 import xpl
    assert xpl.xpl_status_string(0) == b"ok"
    assert b"overlaps" in xpl.xpl_status_string(3)


def test_init_fails_loudly_without_gpu():
    import torch
    if torch.cuda.is_available():
        pytest.skip("a GPU is present")
    from paper_conf_ipps_pirkelbauerlvl20_b200 import xpl
    with pytest.raises(xpl.XplError):
        xpl.Context()

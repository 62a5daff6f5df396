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


def test_binding_struct_layouts_match_the_header(tmp_path):
    """sizeof / offsetof of the report structs added for NEXT-3 / NEXT-4, as the C
    compiler lays them out from include/xpl.h, equal the ctypes mirrors."""
    import subprocess
    from paper_conf_ipps_pirkelbauerlvl20_b200 import xpl
    src = tmp_path / "lay.c"
    src.write_text('#include <stdio.h>\n#include <stddef.h>\n#include "xpl.h"\nint main(void){\n'
                   'printf("%zu %zu %zu %zu %zu %zu\\n", sizeof(xpl_page_report), offsetof(xpl_page_report, flags),'
                   ' sizeof(xpl_launch_record), offsetof(xpl_launch_record, epoch_ms),'
                   ' sizeof(xpl_launch_info), offsetof(xpl_launch_info, shmem));\nreturn 0;}\n')
    exe = tmp_path / "lay"
    subprocess.run(["gcc", "-I", os.path.join(ROOT, "include"), str(src), "-o", str(exe)], check=True)
    got = [int(x) for x in subprocess.run([str(exe)], capture_output=True, text=True, check=True).stdout.split()]
    exp = [ctypes.sizeof(xpl.XplPageReport), xpl.XplPageReport.flags.offset,
           ctypes.sizeof(xpl.XplLaunchRecord), xpl.XplLaunchRecord.epoch_ms.offset,
           ctypes.sizeof(xpl.XplLaunchInfo), xpl.XplLaunchInfo.shmem.offset]
    assert got == exp


def test_um_library_exports_its_header():
    """libxplum.so (CUPTI unified-memory counters, NEXT-4) loads without a GPU and
    exports every function include/xpl_um.h declares."""
    text = re.sub(r"/\*.*?\*/", "", open(os.path.join(ROOT, "include", "xpl_um.h")).read(), flags=re.S)
    names = set(re.findall(r"^\s*\w+\s+(xpl_um_\w+)\s*\(", text, flags=re.M))
    assert {"xpl_um_enable", "xpl_um_disable", "xpl_um_read", "xpl_um_dropped"} <= names
    lib = ctypes.CDLL(os.path.join(ROOT, "paper_conf_ipps_pirkelbauerlvl20_b200", "libxplum.so"))
    assert all(hasattr(lib, n) for n in names)

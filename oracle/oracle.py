"""TEST INFRASTRUCTURE ONLY: ctypes wrapper of liboracle.so (xpl_oracle.cpp).

Replays a trace (xplgen.trace) through the sequential C++ oracle and returns
the rows of every DIAG as dicts.  The header of xpl_oracle.cpp cites the
paper passages each rule follows.
"""
from __future__ import annotations

import ctypes as C
import os
import subprocess

import numpy as np

HERE = os.path.dirname(os.path.abspath(__file__))
LIB = os.path.join(HERE, "liboracle.so")

REPORT_FIELDS = [
    ("id", C.c_uint64), ("base", C.c_uint64), ("bytes", C.c_uint64), ("words", C.c_uint64),
    ("kind", C.c_uint32), ("live", C.c_uint32), ("name_idx", C.c_uint32), ("flags", C.c_uint32),
    ("w_c", C.c_uint64), ("w_g", C.c_uint64), ("r_cc", C.c_uint64), ("r_cg", C.c_uint64),
    ("r_gc", C.c_uint64), ("r_gg", C.c_uint64), ("any_acc", C.c_uint64), ("gpu_acc", C.c_uint64),
    ("alternating", C.c_uint64), ("density_pct_any", C.c_uint64), ("density_pct_gpu", C.c_uint64),
    ("low_density_blocks", C.c_uint64), ("low_density_words", C.c_uint64),
    ("h2d_unused_runs", C.c_uint64), ("h2d_unused_words", C.c_uint64),
    ("d2h_unneeded_runs", C.c_uint64), ("d2h_unneeded_words", C.c_uint64),
    ("ever_accessed", C.c_uint64),
]


class XoReport(C.Structure):
    _fields_ = REPORT_FIELDS


PAGE_FIELDS = [
    ("id", C.c_uint64), ("base", C.c_uint64), ("words", C.c_uint64), ("page_words", C.c_uint64),
    ("pages", C.c_uint64), ("kind", C.c_uint32), ("advice", C.c_uint32), ("cpu_pages", C.c_uint64),
    ("gpu_pages", C.c_uint64), ("shared_pages", C.c_uint64), ("false_shared_pages", C.c_uint64),
    ("alternating_pages", C.c_uint64), ("flags", C.c_uint32), ("pad", C.c_uint32)]


class XoPageReport(C.Structure):
    _fields_ = PAGE_FIELDS


def build():
    """Compile liboracle.so and the CLI with make (plain g++, no CUDA)."""
    subprocess.run(["make", "-s", "-C", HERE], check=True)


_lib = None


def _load():
    global _lib
    if _lib is None:
        if not os.path.exists(LIB):
            build()
        lib = C.CDLL(LIB)
        u64, u32, vp = C.c_uint64, C.c_uint32, C.c_void_p
        lib.xo_new.restype = vp
        lib.xo_delete.argtypes = [vp]
        lib.xo_reg.argtypes = [vp, u64, u64, u32]
        lib.xo_reg.restype = C.c_int64
        lib.xo_free.argtypes = [vp, u64]
        lib.xo_kb.argtypes = [vp]
        lib.xo_ke.argtypes = [vp]
        lib.xo_host.argtypes = [vp, u64, u32, u32]
        lib.xo_dev.argtypes = [vp, u64, u32, u32]
        lib.xo_host_batch.argtypes = [vp, vp, vp, vp, C.c_size_t]
        lib.xo_dev_batch.argtypes = [vp, vp, vp, vp, C.c_size_t]
        lib.xo_copy.argtypes = [vp, u64, u64, u64, u32]
        lib.xo_diag.argtypes = [vp, u32, u64, u64, C.c_int, vp, C.c_size_t, vp, C.c_size_t]
        lib.xo_diag.restype = C.c_int64
        lib.xo_peek.argtypes = [vp, u64, u64]
        lib.xo_pages.argtypes = [vp, u64, vp, C.c_size_t]
        lib.xo_pages.restype = C.c_int64
        lib.xo_advise.argtypes = [vp, u64, u32, C.c_int]
        _lib = lib
    return _lib


def _ptr(a):
    return a.ctypes.data_as(C.c_void_p)


class Oracle:
    """One sequential replay state (xo_state)."""

    def __init__(self):
        self.lib = _load()
        self.s = self.lib.xo_new()

    def close(self):
        if self.s:
            self.lib.xo_delete(self.s)
            self.s = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass

    def _ok(self, rc, op):
        if rc < 0:
            raise RuntimeError(f"oracle rejected {op[0]} (rc={rc})")

    def op(self, op):
        lib, s, t = self.lib, self.s, op[0]
        if t == "REG":
            self._ok(lib.xo_reg(s, op[1], op[2], op[3]), op)
        elif t == "FREE":
            self._ok(lib.xo_free(s, op[1]), op)
        elif t == "KB":
            self._ok(lib.xo_kb(s), op)
        elif t == "KE":
            self._ok(lib.xo_ke(s), op)
        elif t == "H":
            self._ok(lib.xo_host(s, op[1], op[2], op[3]), op)
        elif t == "D":
            self._ok(lib.xo_dev(s, op[1], op[2], op[3]), op)
        elif t in ("HB", "DB"):
            a = np.ascontiguousarray(op[1], dtype=np.uint64)
            z = np.ascontiguousarray(op[2], dtype=np.uint32)
            k = np.ascontiguousarray(op[3], dtype=np.uint8)
            f = lib.xo_host_batch if t == "HB" else lib.xo_dev_batch
            self._ok(f(s, _ptr(a), _ptr(z), _ptr(k), a.size), op)
        elif t == "X":
            self._ok(lib.xo_copy(s, op[2], op[3], op[4], op[1]), op)
        elif t == "DIAG":
            return self.diag(*op[1:6])
        elif t == "PAGES":  # ("PAGES", page_words): the UM page view (NEXT-3)
            return self.pages(op[1])
        elif t == "ADVISE":  # ("ADVISE", ptr, bytes, advice, device)
            self._ok(lib.xo_advise(s, op[1], op[3], op[4]), op)
        else:
            raise ValueError(op)
        return None

    def diag(self, thr, block_words, min_run, reset, names=()):
        names = np.asarray(list(names), dtype=np.uint64)
        cap = 64
        while True:
            out = (XoReport * cap)()
            n = self.lib.xo_diag(self.s, thr, block_words, min_run, int(reset),
                                 _ptr(names) if names.size else None, names.size, out, cap)
            if n < 0:
                raise RuntimeError("oracle rejected DIAG")
            if n <= cap:
                return [{f: getattr(out[i], f) for f, _ in REPORT_FIELDS} for i in range(n)]
            cap = n

    def pages(self, page_words):
        cap = 64
        while True:
            out = (XoPageReport * cap)()
            n = self.lib.xo_pages(self.s, page_words, out, cap)
            if n < 0:
                raise RuntimeError("oracle rejected PAGES")
            if n <= cap:
                return [{f: getattr(out[i], f) for f, _ in PAGE_FIELDS if f != "pad"} for i in range(n)]
            cap = n

    def peek(self, alloc_id, word):
        return self.lib.xo_peek(self.s, alloc_id, word)


def run_trace(ops):
    """Replay a whole trace; return the list of DIAG results (each a list of row dicts)."""
    o = Oracle()
    res = []
    for op in ops:
        r = o.op(op)
        if r is not None:
            res.append(r)
    o.close()
    return res

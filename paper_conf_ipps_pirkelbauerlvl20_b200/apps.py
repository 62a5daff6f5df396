"""Binding of the instrumented workload applications in libxplwork.so (xplw.h).

Allocates each app's arrays (device arena in HBM via torch, host arena pinned),
runs the native C++ program through ctypes and returns its reports.  The apps
call the C-ABI themselves; this module only marshals.
"""
from __future__ import annotations

import ctypes as C

import numpy as np

from . import xpl
from .xpl import REPORT_FIELDS, XplAllocReport, XplDiagParams

u64, u32, i32, vp, sz = C.c_uint64, C.c_uint32, C.c_int, C.c_void_p, C.c_size_t
MAXA = 64


class XplwArrays(C.Structure):
    _fields_ = [("addr", u64 * MAXA), ("bytes", u64 * MAXA), ("kind", u32 * MAXA), ("n", i32)]


class XplwRun(C.Structure):
    _fields_ = [("ctx", vp), ("stream", vp), ("do_copies", i32), ("diag_each", i32),
                ("params", XplDiagParams), ("out", vp), ("out_cap", sz), ("n_out", sz),
                ("diag_rows", vp), ("diag_cap", sz), ("n_diag", sz), ("dev_accesses", u64),
                ("host_accesses", u64), ("copy_words", u64), ("epochs", u64), ("status", i32),
                ("time_kernels", i32), ("kernel_ms", C.c_double), ("host_ms", C.c_double),
                ("diag_no_reset", i32), ("keep_allocs", i32), ("rank", i32), ("world", i32),
                ("kernel_ms_each", vp), ("kernel_cap", sz)]


_w = xpl._work
_w.xplw_hotspot.argtypes = [C.POINTER(XplwRun), C.POINTER(XplwArrays), i32, i32, i32]
_w.xplw_backprop.argtypes = [C.POINTER(XplwRun), C.POINTER(XplwArrays), i32, i32]
_w.xplw_bfs.argtypes = [C.POINTER(XplwRun), C.POINTER(XplwArrays), i32, i32, vp, C.POINTER(i32)]
_w.xplw_nw.argtypes = [C.POINTER(XplwRun), C.POINTER(XplwArrays), i32, i32, vp]
_w.xplw_sw.argtypes = [C.POINTER(XplwRun), C.POINTER(XplwArrays), i32, i32, i32, i32, i32, C.POINTER(i32)]
_w.xplw_lulesh.argtypes = [C.POINTER(XplwRun), C.POINTER(XplwArrays), i32, i32, vp, vp]
_w.xplw_lulesh_layout.argtypes = [i32]
_w.xplw_lulesh_layout.restype = i32
_w.xplw_alloc_managed.argtypes = [u64]
_w.xplw_alloc_managed.restype = vp
_w.xplw_free_managed.argtypes = [vp]
_w.xplw_memcpy_async.argtypes = [vp, vp, u64, vp]
_w.xplw_memcpy_async.restype = i32
for f in ("xplw_hotspot", "xplw_backprop", "xplw_bfs", "xplw_nw", "xplw_sw", "xplw_free_managed", "xplw_lulesh"):
    getattr(_w, f).restype = i32


class Arena:
    """Device + pinned-host memory for one app, laid out by xplgen.rodinia.layout."""

    def __init__(self, spec):
        import torch
        from xplgen.rodinia import arena_sizes, layout
        sz = arena_sizes(spec)
        self.dev = torch.empty(sz["dev"] + 4096, dtype=torch.uint8, device="cuda")
        self.host = torch.empty(sz["host"] + 4096, dtype=torch.uint8).pin_memory()
        self.managed = None
        self.managed_bytes = sz["managed"]
        mb = 0
        if sz["managed"]:
            self.managed = _w.xplw_alloc_managed(sz["managed"] + 4096)
            if not self.managed:
                raise MemoryError("cudaMallocManaged failed")
            mb = (self.managed + 4095) // 4096 * 4096
        db = (self.dev.data_ptr() + 4095) // 4096 * 4096
        hb = (self.host.data_ptr() + 4095) // 4096 * 4096
        self.addrs, _, _ = layout(spec, db, hb, mb)
        self.spec = spec
        self.arrays = XplwArrays()
        for i, (a, s) in enumerate(zip(self.addrs, spec)):
            self.arrays.addr[i] = a
            self.arrays.bytes[i] = s[1]
            self.arrays.kind[i] = s[2]
        self.arrays.n = len(spec)

    def __del__(self):
        if getattr(self, "managed", None):
            _w.xplw_free_managed(self.managed)
            self.managed = None

    def view(self, name):
        """numpy view (uint8) of one array by name (host, managed) or torch view (device)."""
        for a, sp in zip(self.addrs, self.spec):
            if sp[0] == name:
                if sp[3] == "managed":
                    return np.ctypeslib.as_array((C.c_uint8 * sp[1]).from_address(a))
                if sp[3] == "host":
                    o = a - self.host.data_ptr()
                    return self.host.numpy()[o:o + sp[1]]
                o = a - self.dev.data_ptr()
                return self.dev[o:o + sp[1]]
        raise KeyError(name)

    def host_views(self):
        """numpy views of the host arrays (for seeding inputs)."""
        base = self.host.data_ptr()
        hv = self.host.numpy()
        out = []
        for a, s in zip(self.addrs, self.spec):
            if s[3] == "host":
                o = a - base
                out.append(hv[o:o + s[1]])
        return out


class Run:
    """One xplw_run: the context (or None = uninstrumented twin) and outputs."""

    def __init__(self, ctx, stream, do_copies=False, diag_each=True, params=(50, 0, 256), out_cap=4096,
                 time_kernels=False, diag_reset=True, keep_allocs=False, rank=0, world=1):
        self.r = XplwRun()
        self.r.rank, self.r.world = rank, world
        if time_kernels:  # each launch's event time too (LULESH)
            self.kernel_each = (C.c_float * 8192)()
            self.r.kernel_ms_each = C.cast(self.kernel_each, vp)
            self.r.kernel_cap = 8192
        self.r.diag_no_reset = int(not diag_reset)
        self.r.keep_allocs = int(keep_allocs)
        self.r.time_kernels = int(time_kernels)
        self.r.ctx = ctx.h if ctx is not None else None
        self.r.stream = stream
        self.r.do_copies = int(do_copies)
        self.r.diag_each = int(diag_each)
        self.r.params = XplDiagParams(*params)
        self.out = (XplAllocReport * out_cap)()
        self.rows = (u32 * 4096)()
        self.r.out = C.cast(self.out, vp)
        self.r.out_cap = out_cap
        self.r.diag_rows = C.cast(self.rows, vp)
        self.r.diag_cap = 4096

    def reports(self):
        """The diagnoses of the run, each a list of row dicts."""
        res, k = [], 0
        for d in range(self.r.n_diag):
            n = self.rows[d]
            res.append([{f: getattr(self.out[k + i], f) for f, _ in REPORT_FIELDS} for i in range(n)])
            k += n
        return res

    def check(self):
        if self.r.status:
            raise xpl.XplError("workload", self.r.status)


def hotspot(run: Run, arena: Arena, rows, cols, iters):
    st = _w.xplw_hotspot(C.byref(run.r), C.byref(arena.arrays), rows, cols, iters)
    run.check()
    return st


def backprop(run: Run, arena: Arena, n_in, hid):
    st = _w.xplw_backprop(C.byref(run.r), C.byref(arena.arrays), n_in, hid)
    run.check()
    return st


def bfs(run: Run, arena: Arena, n, deg, hook_counter):
    """hook_counter: a torch int64 cuda tensor of 1 element (the kernels add to it)."""
    lv = i32(0)
    st = _w.xplw_bfs(C.byref(run.r), C.byref(arena.arrays), n, deg, hook_counter.data_ptr(), C.byref(lv))
    run.check()
    return lv.value


def bfs_prepare(arena: Arena, n, deg, edges, resident: bool):
    """Inputs of one bfs run: the graph in h_edges; for resident-data runs also the
    device arrays as the program's H2D copies would have left them."""
    import torch
    from xplgen.rodinia import bfs_device_initial
    arena.view("h_edges").view(np.int32)[:] = edges
    if resident:
        for name, arr in bfs_device_initial(n, deg, edges).items():
            arena.view(name).copy_(torch.from_numpy(arr.view(np.uint8)), non_blocking=False)


def nw(run: Run, arena: Arena, n, penalty, blosum):
    """blosum: numpy int32 (24, 24), contiguous."""
    st = _w.xplw_nw(C.byref(run.r), C.byref(arena.arrays), n, penalty, blosum.ctypes.data)
    run.check()
    return st


def sw(run: Run, arena: Arena, n, m, per_diagonal, tb_every, diag_every, inp):
    """Smith-Waterman (managed arrays a, b, H); inp = xplgen.sw.sw_inputs().
    Returns the traceback length."""
    import torch
    arena.view("a").view(np.int32)[:] = inp["a"]
    arena.view("b").view(np.int32)[:] = inp["b"]
    torch.cuda.synchronize()
    tb = i32(0)
    _w.xplw_sw(C.byref(run.r), C.byref(arena.arrays), n, m, int(per_diagonal), tb_every, diag_every,
               C.byref(tb))
    run.check()
    return tb.value


def lulesh_prepare(arena: Arena, s, topo):
    """Write the mesh topology (input) into the managed topology arrays."""
    import torch
    from xplgen import lulesh as L
    for k, arr in topo.items():
        arena.view(L.NAMES[k]).view(np.int32)[:] = arr
    torch.cuda.synchronize()


def lulesh_topology_host(topo):
    """Pinned host copies of the mesh topology (the e2e input upload's source)."""
    import torch
    return {k: torch.from_numpy(np.ascontiguousarray(v)).pin_memory() for k, v in topo.items()}


def lulesh_upload(arena: Arena, host_topo, stream):
    """Upload the topology from pinned host memory into the managed arrays on
    `stream` (cudaMemcpyAsync); returns the bytes copied."""
    from xplgen import lulesh as L
    nb = 0
    for k, t in host_topo.items():
        a = arena.addrs[[sp[0] for sp in arena.spec].index(L.NAMES[k])]
        n = t.numel() * t.element_size()
        if _w.xplw_memcpy_async(a, t.data_ptr(), n, stream):
            raise xpl.XplError("cudaMemcpyAsync", 6)
        nb += n
    return nb


def lulesh(run: Run, arena: Arena, s, steps, hook_counter):
    """Returns the temporaries' addresses [(force, gradient)] per step."""
    tmp = (u64 * (2 * steps))()
    _w.xplw_lulesh(C.byref(run.r), C.byref(arena.arrays), s, steps, hook_counter.data_ptr(), tmp)
    run.check()
    return [(tmp[2 * i], tmp[2 * i + 1]) for i in range(steps)]


def lulesh_layout():
    """The CUDA program's domain layout (for the cross-check with xplgen.lulesh)."""
    return [_w.xplw_lulesh_layout(i) for i in range(9)]

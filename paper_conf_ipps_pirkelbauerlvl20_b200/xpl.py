"""ctypes binding of include/xpl.h (libxpl.so) and of the instrumented user
kernels in libxplwork.so.  Marshalling only; names follow the C-ABI.

Fails loudly (ImportError/OSError) if the shared libraries are missing: there
is no fallback path.
"""
from __future__ import annotations

import ctypes as C
import os

import numpy as np

from . import LIB_PATH, WORK_PATH

if not os.path.exists(LIB_PATH):
    raise ImportError(f"{LIB_PATH} is not built: run __graft_entry__.build() (no CPU fallback exists)")

_lib = C.CDLL(LIB_PATH, mode=C.RTLD_GLOBAL)
_work = C.CDLL(WORK_PATH) if os.path.exists(WORK_PATH) else None

u64, u32, i32, vp, sz = C.c_uint64, C.c_uint32, C.c_int, C.c_void_p, C.c_size_t

XPL_OK = 0
STATUS = {0: "XPL_OK", 1: "XPL_ERR_INVALID_ARG", 2: "XPL_ERR_OOM", 3: "XPL_ERR_OVERLAP",
          4: "XPL_ERR_UNKNOWN_PTR", 5: "XPL_ERR_STATE", 6: "XPL_ERR_CUDA", 7: "XPL_ERR_NCCL",
          8: "XPL_ERR_DEVICE_OVERFLOW"}
ALLOC_DEVICE, ALLOC_MANAGED, ALLOC_HOST = 0, 1, 2
ACC_R, ACC_W, ACC_RW = 1, 2, 3
COPY_H2D, COPY_D2H, COPY_H2H, COPY_D2D, MEMSET_DEV = 0, 1, 2, 3, 4

HOST_ACCESS_DTYPE = np.dtype([("addr", "<u8"), ("size", "<u4"), ("kind", "<u4")])
HOST_STRIDED_DTYPE = np.dtype([("addr", "<u8"), ("size", "<u4"), ("kind", "<u4"), ("stride", "<i8"),
                               ("count", "<u8")])


_ALLGATHER = C.CFUNCTYPE(i32, vp, vp, C.c_size_t, vp)
_ALLTOALLV = C.CFUNCTYPE(i32, vp, vp, C.POINTER(u64), vp, C.POINTER(u64))
_BARRIER = C.CFUNCTYPE(i32, vp)


class XplComm(C.Structure):
    """xpl_comm: the collectives of a sharded context (host buffers, blocking)."""
    _fields_ = [("user", vp), ("allgather", _ALLGATHER), ("alltoallv", _ALLTOALLV), ("barrier", _BARRIER)]


class XplConfig(C.Structure):
    _fields_ = [("device", i32), ("rank", i32), ("world", i32), ("comm", C.POINTER(XplComm)),
                ("pool_words", u64), ("staging_recs", u64), ("max_rows", u32)]


class XplDiagParams(C.Structure):
    _fields_ = [("density_threshold_pct", u32), ("block_words", u64), ("min_run_words", u64)]


class XplName(C.Structure):
    _fields_ = [("addr", vp), ("expr", C.c_char_p), ("elem_size", u32)]


REPORT_FIELDS = [
    ("id", u64), ("base", u64), ("bytes", u64), ("words", u64),
    ("kind", u32), ("live", u32), ("name_idx", u32), ("flags", u32),
    ("w_c", u64), ("w_g", u64), ("r_cc", u64), ("r_cg", u64), ("r_gc", u64), ("r_gg", u64),
    ("any_acc", u64), ("gpu_acc", u64), ("alternating", u64),
    ("density_pct_any", u64), ("density_pct_gpu", u64),
    ("low_density_blocks", u64), ("low_density_words", u64),
    ("h2d_unused_runs", u64), ("h2d_unused_words", u64),
    ("d2h_unneeded_runs", u64), ("d2h_unneeded_words", u64), ("ever_accessed", u64),
]


class XplAllocReport(C.Structure):
    _fields_ = REPORT_FIELDS


REPORT_BYTES = C.sizeof(XplAllocReport)


class XplPartial(C.Structure):
    _fields_ = [("logical_id", u64), ("word_offset", u64), ("words", u64), ("logical_words", u64),
                ("logical_bytes", u64), ("base", u64), ("kind", u32), ("live", u32), ("name_idx", u32),
                ("pad", u32), ("cnt", u64 * 9), ("u_run", u64 * 5), ("d_run", u64 * 5),
                ("low_density_blocks", u64), ("low_density_words", u64), ("blk_first", u64),
                ("blk_first_g", u64), ("blk_first_s", u64), ("blk_last", u64), ("blk_last_g", u64),
                ("blk_last_s", u64), ("ever_accessed", u64)]


class XplStats(C.Structure):
    _fields_ = [(n, u64) for n in ("epochs", "folds", "fold_chunks", "host_records",
                                   "host_records_packed", "merge_segments", "range_segments",
                                   "diagnoses", "fold_chunks_max", "kernel_launches")]


class XplDevCtx(C.Structure):
    _fields_ = [("rows", vp), ("n_rows", vp), ("pool", vp), ("cmap", vp), ("smap", vp), ("n_super", vp),
                ("flags", vp)]


def _sig(name, args, res=i32, lib=_lib):
    f = getattr(lib, name)
    f.argtypes = args
    f.restype = res
    return f


xpl_init = _sig("xpl_init", [C.POINTER(XplConfig), C.POINTER(vp)])
xpl_finalize = _sig("xpl_finalize", [vp])
xpl_register_alloc = _sig("xpl_register_alloc", [vp, vp, sz, i32])
xpl_free = _sig("xpl_free", [vp, vp])
xpl_kernel_begin = _sig("xpl_kernel_begin", [vp, vp])
xpl_kernel_end = _sig("xpl_kernel_end", [vp, vp])
xpl_record_host = _sig("xpl_record_host", [vp, vp, sz])
xpl_record_host_ranges = _sig("xpl_record_host_ranges", [vp, vp, sz])
xpl_record_host_strided = _sig("xpl_record_host_strided", [vp, vp, sz])
xpl_record_copy = _sig("xpl_record_copy", [vp, vp, vp, sz, i32])
xpl_diagnose = _sig("xpl_diagnose", [vp, C.POINTER(XplDiagParams), C.POINTER(XplName), sz,
                                     C.POINTER(XplAllocReport), sz, C.POINTER(sz), i32])
xpl_register_alloc_piece = _sig("xpl_register_alloc_piece", [vp, vp, sz, i32, u64, u64, u64])
xpl_diagnose_partials = _sig("xpl_diagnose_partials", [vp, C.POINTER(XplDiagParams), C.POINTER(XplName), sz,
                                                       C.POINTER(XplPartial), sz, C.POINTER(sz), i32])
xpl_combine_partials = _sig("xpl_combine_partials", [C.POINTER(XplPartial), sz, C.POINTER(XplDiagParams),
                                                     C.POINTER(XplAllocReport), sz, C.POINTER(sz)])
xpl_format_reports = _sig("xpl_format_reports", [C.POINTER(XplAllocReport), sz, C.POINTER(XplName), sz, i32,
                                                 i32, C.c_char_p, sz, C.POINTER(sz)])
xpl_get_device_ctx = _sig("xpl_get_device_ctx", [vp, C.POINTER(XplDevCtx)])
xpl_release_stream = _sig("xpl_release_stream", [vp, vp])
xpl_comm_nccl_unique_id = _sig("xpl_comm_nccl_unique_id", [vp])
xpl_comm_nccl_create = _sig("xpl_comm_nccl_create", [vp, i32, i32, i32, C.POINTER(C.POINTER(XplComm))])
xpl_comm_nccl_destroy = _sig("xpl_comm_nccl_destroy", [C.POINTER(XplComm)])
xpl_shadow_dump = _sig("xpl_shadow_dump", [vp, vp, u64, u64, vp])
PAGE_REPORT_FIELDS = [
    ("id", u64), ("base", u64), ("words", u64), ("page_words", u64), ("pages", u64),
    ("kind", u32), ("advice", u32), ("cpu_pages", u64), ("gpu_pages", u64), ("shared_pages", u64),
    ("false_shared_pages", u64), ("alternating_pages", u64), ("flags", u32), ("pad", u32)]


class XplPageReport(C.Structure):
    _fields_ = PAGE_REPORT_FIELDS


xpl_page_summary = _sig("xpl_page_summary", [vp, u64, C.POINTER(XplPageReport), sz, C.POINTER(sz)])
xpl_page_flags = _sig("xpl_page_flags", [vp, vp, u64, vp, u64])
xpl_mem_advise = _sig("xpl_mem_advise", [vp, vp, sz, i32, i32])


class XplLaunchInfo(C.Structure):
    _fields_ = [("name", C.c_char_p), ("grid", u32 * 3), ("block", u32 * 3), ("shmem", u32)]


class XplLaunchRecord(C.Structure):
    _fields_ = [("seq", u64), ("epoch", u64), ("stream", u64), ("grid", u32 * 3), ("block", u32 * 3),
                ("shmem", u32), ("name_idx", u32), ("threads", u64), ("launches_in_epoch", u64),
                ("epoch_written_chunks", u64), ("epoch_ms", C.c_double)]


xpl_launch_log_enable = _sig("xpl_launch_log_enable", [vp, i32])
xpl_kernel_launch = _sig("xpl_kernel_launch", [vp, vp, C.POINTER(XplLaunchInfo)])
xpl_launch_log = _sig("xpl_launch_log", [vp, C.POINTER(XplLaunchRecord), sz, C.POINTER(sz), i32])
xpl_launch_name = _lib.xpl_launch_name
xpl_launch_name.argtypes = [vp, u32]
xpl_launch_name.restype = C.c_char_p
xpl_flush = _sig("xpl_flush", [vp])
xpl_sync = _sig("xpl_sync", [vp])
xpl_join = _sig("xpl_join", [vp, vp])
xpl_runtime_stream = _sig("xpl_runtime_stream", [vp, C.POINTER(vp)])
xpl_get_stats = _sig("xpl_get_stats", [vp, C.POINTER(XplStats)])
xpl_status_string = _sig("xpl_status_string", [i32], C.c_char_p)
xpl_profile = _sig("xpl_profile", [vp, i32])


class XplKernelTime(C.Structure):
    _fields_ = [("launches", u64), ("ms", C.c_double), ("bytes", u64)]


KERNEL_CLASSES = ["fold", "merge", "range", "diag_tile", "diagnose", "pages"]
xpl_profile_read = _sig("xpl_profile_read", [vp, C.POINTER(XplKernelTime), i32])

EXPORTED = ["xpl_init", "xpl_finalize", "xpl_register_alloc", "xpl_free", "xpl_kernel_begin",
            "xpl_kernel_end", "xpl_record_host", "xpl_record_host_ranges", "xpl_record_host_strided", "xpl_record_copy", "xpl_diagnose",
            "xpl_get_device_ctx", "xpl_shadow_dump", "xpl_flush", "xpl_sync", "xpl_join",
            "xpl_runtime_stream", "xpl_get_stats", "xpl_status_string", "xpl_profile",
            "xpl_profile_read", "xpl_register_alloc_piece", "xpl_diagnose_partials", "xpl_combine_partials",
            "xpl_format_reports", "xpl_page_summary", "xpl_page_flags", "xpl_mem_advise",
            "xpl_launch_log_enable", "xpl_kernel_launch", "xpl_launch_log", "xpl_launch_name",
            "xpl_release_stream", "xpl_comm_nccl_unique_id", "xpl_comm_nccl_create",
            "xpl_comm_nccl_destroy"]

if _work is not None:
    xplw_bind = _sig("xplw_bind", [vp], lib=_work)
    xplw_replay = _sig("xplw_replay", [vp, vp, vp, u64, i32, i32, vp], lib=_work)
    xplw_replay_traced = _sig("xplw_replay_traced", [vp, vp, vp, vp, u64, i32, i32, vp], lib=_work)
    xplw_replay_split = _sig("xplw_replay_split", [vp, vp, vp, vp, i32, i32, i32, vp], lib=_work)
    xplw_atomic_bench = _sig("xplw_atomic_bench", [vp, u64, i32, vp], lib=_work)
    xplw_touch = _sig("xplw_touch", [u64, u64, u32, vp, u64], lib=_work)
    xplw_stream = _sig("xplw_stream", [vp, vp, u64, i32, i32, vp], lib=_work)
    xplw_replay_k = _sig("xplw_replay_k", [vp, vp, u64, i32, i32, i32, vp], lib=_work)
    xplw_handle_replay = _sig("xplw_handle_replay", [u64, i32, vp, u64, i32, i32, i32, vp], lib=_work)
    # (optional so that A/B builds of the workload library without it still load)
    xplw_read_lat = (_sig("xplw_read_lat", [vp, u64, i32, i32, i32, vp], lib=_work)
                     if hasattr(_work, "xplw_read_lat") else None)


class XplError(RuntimeError):
    def __init__(self, fn, status):
        super().__init__(f"{fn} -> {STATUS.get(status, status)}")
        self.status = status


def check(fn, status):
    if status != XPL_OK:
        raise XplError(fn, status)


class TorchComm:
    """xpl_comm over a torch.distributed process group (argument marshalling
    only: the runtime calls these from xpl_init / collective calls).  Host
    tensors, so any backend works (gloo in the tests; use NcclComm on GPUs)."""

    def __init__(self, group=None):
        import torch.distributed as dist
        self.dist, self.group = dist, group
        self.world = dist.get_world_size(group)
        self.rank = dist.get_rank(group)
        self._cb = (_ALLGATHER(self._allgather), _ALLTOALLV(self._alltoallv), _BARRIER(self._barrier))
        self.c = XplComm(None, *self._cb)

    def _gather_bytes(self, data):
        import torch
        n = torch.tensor([len(data)], dtype=torch.int64)
        ns = [torch.zeros(1, dtype=torch.int64) for _ in range(self.world)]
        self.dist.all_gather(ns, n, group=self.group)
        m = max(int(x.item()) for x in ns)
        t = torch.zeros(max(m, 1), dtype=torch.uint8)
        if data:
            t[:len(data)] = torch.frombuffer(bytearray(data), dtype=torch.uint8)
        outs = [torch.zeros(max(m, 1), dtype=torch.uint8) for _ in range(self.world)]
        self.dist.all_gather(outs, t, group=self.group)
        return [bytes(o[:int(k.item())].numpy()) for o, k in zip(outs, ns)]

    def _allgather(self, user, send, nbytes, recv):
        try:
            parts = self._gather_bytes(C.string_at(send, nbytes) if nbytes else b"")
            C.memmove(recv, b"".join(parts), nbytes * self.world)
            return 0
        except Exception:  # noqa: BLE001 (reported to the runtime as a failed collective)
            return 1

    def _alltoallv(self, user, send, sb, recv, rb):
        """All-to-all as two all-gathers (the send sizes, then the send
        buffers): each rank cuts its part out of every rank's buffer."""
        try:
            import numpy as np
            R = self.world
            tot = sum(sb[q] for q in range(R))
            blobs = self._gather_bytes(C.string_at(send, tot) if tot else b"")
            sz = np.frombuffer(b"".join(self._gather_bytes(np.array([sb[q] for q in range(R)], np.uint64).tobytes())),
                               np.uint64).reshape(R, R)
            mine = b"".join(blobs[q][int(sz[q, :self.rank].sum()):int(sz[q, :self.rank + 1].sum())] for q in range(R))
            if len(mine) != sum(rb[q] for q in range(R)):
                return 2
            if mine:
                C.memmove(recv, mine, len(mine))
            return 0
        except Exception:  # noqa: BLE001
            return 1

    def _barrier(self, user):
        try:
            self.dist.barrier(group=self.group)
            return 0
        except Exception:  # noqa: BLE001
            return 1


class NcclComm:
    """xpl_comm over NCCL (libxpl.so's own, xpl_comm_nccl_create): rank 0's
    unique id reaches the others through `broadcast_id(bytes) -> bytes`."""

    def __init__(self, rank, world, device, broadcast_id):
        uid = (C.c_uint8 * 128)()
        if rank == 0:
            check("xpl_comm_nccl_unique_id", xpl_comm_nccl_unique_id(uid))
        got = broadcast_id(bytes(uid))
        C.memmove(uid, got, 128)
        p = C.POINTER(XplComm)()
        check("xpl_comm_nccl_create", xpl_comm_nccl_create(uid, rank, world, device, C.byref(p)))
        self.p, self.rank, self.world = p, rank, world

    def close(self):
        if self.p:
            check("xpl_comm_nccl_destroy", xpl_comm_nccl_destroy(self.p))
            self.p = None


class Context:
    """One xpl_ctx (one process, one GPU).  comm (TorchComm / NcclComm) with
    world > 1: a sharded context (COLLECTIVE calls, include/xpl.h)."""

    def __init__(self, device=0, pool_words=0, staging_recs=0, max_rows=0, comm=None):
        self.comm = comm  # (kept alive: the runtime holds its pointer)
        if comm is None:
            cfg = XplConfig(device, 0, 1, None, pool_words, staging_recs, max_rows)
        else:
            cp = C.pointer(comm.c) if isinstance(comm, TorchComm) else comm.p
            cfg = XplConfig(device, comm.rank, comm.world, cp, pool_words, staging_recs, max_rows)
        h = vp()
        check("xpl_init", xpl_init(C.byref(cfg), C.byref(h)))
        self.h = h
        if _work is not None:
            check("xplw_bind", xplw_bind(self.h))

    def bind(self):
        """Point the instrumented kernels of libxplwork at this context."""
        check("xplw_bind", xplw_bind(self.h))

    def close(self):
        if self.h:
            xpl_finalize(self.h)
            self.h = None

    def __enter__(self):
        return self

    def __exit__(self, *a):
        self.close()

    def register(self, ptr, nbytes, kind):
        check("xpl_register_alloc", xpl_register_alloc(self.h, ptr, nbytes, kind))

    def free(self, ptr):
        check("xpl_free", xpl_free(self.h, ptr))

    def kernel_begin(self, stream=0):
        check("xpl_kernel_begin", xpl_kernel_begin(self.h, stream))

    def kernel_end(self, stream=0):
        check("xpl_kernel_end", xpl_kernel_end(self.h, stream))

    def record_host(self, recs: np.ndarray):
        recs = np.ascontiguousarray(recs, dtype=HOST_ACCESS_DTYPE)
        check("xpl_record_host", xpl_record_host(self.h, recs.ctypes.data, recs.size))

    def record_host_ranges(self, recs: np.ndarray):
        recs = np.ascontiguousarray(recs, dtype=HOST_ACCESS_DTYPE)
        check("xpl_record_host_ranges", xpl_record_host_ranges(self.h, recs.ctypes.data, recs.size))

    def record_host_strided(self, recs: np.ndarray):
        """recs: HOST_STRIDED_DTYPE records (addr, size, kind, stride, count)."""
        recs = np.ascontiguousarray(recs, dtype=HOST_STRIDED_DTYPE)
        check("xpl_record_host_strided", xpl_record_host_strided(self.h, recs.ctypes.data, recs.size))

    def record_copy(self, dst, src, nbytes, direction):
        check("xpl_record_copy", xpl_record_copy(self.h, dst, src, nbytes, direction))

    def diagnose(self, thr=50, block_words=0, min_run=256, reset=True, names=()):
        p = XplDiagParams(thr, block_words, min_run)
        nn = len(names)
        arr = (XplName * max(nn, 1))()
        for i, a in enumerate(names):
            arr[i].addr = a
            arr[i].expr = b""
            arr[i].elem_size = 0
        cap = 64
        while True:
            out = (XplAllocReport * cap)()
            n = sz(0)
            st = xpl_diagnose(self.h, C.byref(p), arr if nn else None, nn, out, cap, C.byref(n),
                              int(bool(reset)))
            if st == 1 and n.value > cap:
                cap = n.value
                continue
            check("xpl_diagnose", st)
            return [{f: getattr(out[i], f) for f, _ in REPORT_FIELDS} for i in range(n.value)]

    def register_piece(self, ptr, nbytes, kind, logical_id, word_offset, logical_bytes):
        check("xpl_register_alloc_piece",
              xpl_register_alloc_piece(self.h, ptr, nbytes, kind, logical_id, word_offset, logical_bytes))

    def diagnose_partials(self, thr=50, block_words=0, min_run=256, reset=True):
        """This context's partials as raw bytes (what ranks exchange)."""
        p = XplDiagParams(thr, block_words, min_run)
        cap = 64
        while True:
            out = (XplPartial * cap)()
            n = sz(0)
            st = xpl_diagnose_partials(self.h, C.byref(p), None, 0, out, cap, C.byref(n), int(bool(reset)))
            if st == 1 and n.value > cap:
                cap = n.value
                continue
            check("xpl_diagnose_partials", st)
            return bytes(memoryview(out).cast("B")[:n.value * C.sizeof(XplPartial)])

    def page_summary(self, page_words=1024):
        """The UM page view of every live row (xpl_page_summary), as dicts."""
        cap = 64
        while True:
            out = (XplPageReport * cap)()
            n = sz(0)
            st = xpl_page_summary(self.h, page_words, out, cap, C.byref(n))
            if st == 1 and n.value > cap:
                cap = n.value
                continue
            check("xpl_page_summary", st)
            return [{f: getattr(out[i], f) for f, _ in PAGE_REPORT_FIELDS if f != "pad"} for i in range(n.value)]

    def page_flags(self, base, page_words, n_pages):
        out = np.zeros(max(1, n_pages), dtype=np.uint8)
        check("xpl_page_flags", xpl_page_flags(self.h, base, page_words, out.ctypes.data, n_pages))
        return out[:n_pages]

    def mem_advise(self, ptr, nbytes, advice, device=0):
        check("xpl_mem_advise", xpl_mem_advise(self.h, ptr, nbytes, advice, device))

    def launch_log_enable(self, enable=True):
        check("xpl_launch_log_enable", xpl_launch_log_enable(self.h, int(bool(enable))))

    def kernel_launch(self, stream, name, grid, block, shmem=0):
        """Log one launch of the open epoch (xpl_kernel_launch)."""
        g = tuple(grid) + (1,) * (3 - len(grid))
        b = tuple(block) + (1,) * (3 - len(block))
        li = XplLaunchInfo(name.encode() if name is not None else None, (u32 * 3)(*g), (u32 * 3)(*b), shmem)
        check("xpl_kernel_launch", xpl_kernel_launch(self.h, stream, C.byref(li)))

    def launch_log(self, reset=True):
        """The launch log (xpl_launch_log) as dicts, names resolved."""
        cap = 256
        while True:
            out = (XplLaunchRecord * cap)()
            n = sz(0)
            st = xpl_launch_log(self.h, out, cap, C.byref(n), int(bool(reset)))
            if st == 1 and n.value > cap:
                cap = n.value
                continue
            check("xpl_launch_log", st)
            res = []
            for i in range(n.value):
                r = out[i]
                d = {f: getattr(r, f) for f, _ in XplLaunchRecord._fields_}
                d["grid"], d["block"] = tuple(r.grid), tuple(r.block)
                nm = xpl_launch_name(self.h, r.name_idx)
                d["name"] = nm.decode() if nm is not None else None
                res.append(d)
            return res

    def replay_traced(self, d_addr, d_size, d_acc, n, grid=0, block=256, stream=0):
        """The replay kernel launched through the kernel-launch wrapper
        (xpl_trace_kernel_launch: its own or a nested epoch, logged)."""
        if grid <= 0:
            grid = max(1, min((n + block - 1) // block, 148 * 8))
        check("xplw_replay_traced", xplw_replay_traced(self.h, d_addr, d_size, d_acc, n, grid, block, stream))

    def shadow_dump(self, base, word0, n):
        out = np.zeros(n, dtype=np.uint8)
        check("xpl_shadow_dump", xpl_shadow_dump(self.h, base, word0, n, out.ctypes.data))
        return out

    def flush(self):
        check("xpl_flush", xpl_flush(self.h))

    def sync(self):
        check("xpl_sync", xpl_sync(self.h))

    def join(self, stream):
        """Make `stream` wait (on the device) for all runtime work enqueued so far."""
        check("xpl_join", xpl_join(self.h, stream))

    def release_stream(self, stream):
        """The runtime stops using `stream` (before the caller destroys it)."""
        check("xpl_release_stream", xpl_release_stream(self.h, stream))

    def runtime_stream(self):
        s = vp()
        check("xpl_runtime_stream", xpl_runtime_stream(self.h, C.byref(s)))
        return s.value or 0

    def stats(self):
        s = XplStats()
        check("xpl_get_stats", xpl_get_stats(self.h, C.byref(s)))
        return {f: getattr(s, f) for f, _ in XplStats._fields_}

    def profile(self, enable=True):
        check("xpl_profile", xpl_profile(self.h, int(bool(enable))))

    def profile_read(self, reset=True):
        arr = (XplKernelTime * len(KERNEL_CLASSES))()
        check("xpl_profile_read", xpl_profile_read(self.h, arr, int(bool(reset))))
        return {k: {"launches": arr[i].launches, "ms": arr[i].ms, "bytes": arr[i].bytes}
                for i, k in enumerate(KERNEL_CLASSES)}

    def device_ctx(self):
        d = XplDevCtx()
        check("xpl_get_device_ctx", xpl_get_device_ctx(self.h, C.byref(d)))
        return d

    def touch(self, base, nwords, seed=1, stream=0, i0=0):
        """Launch the synthetic instrumented touch kernel (libxplwork) over nwords at
        base = logical words i0 .. i0+nwords-1 of its access pattern."""
        check("xplw_touch", xplw_touch(base, nwords, seed, stream, i0))

    def replay(self, d_addr, d_size, d_acc, n, grid=0, block=256, stream=0):
        """Launch the instrumented replay kernel (libxplwork) on device arrays."""
        if grid <= 0:
            grid = max(1, min((n + block - 1) // block, 148 * 8))
        check("xplw_replay", xplw_replay(d_addr, d_size, d_acc, n, grid, block, stream))

    def replay_k(self, d_addr, d_size, n, kind, grid=0, block=256, stream=0):
        """The replay kernel with one compile-time access kind for all n events."""
        if grid <= 0:
            grid = max(1, min((n + block - 1) // block, 148 * 8))
        check("xplw_replay_k", xplw_replay_k(d_addr, d_size, n, kind, grid, block, stream))

    def replay_split(self, d_addr, d_size, d_acc, d_seg, nseg, grid=0, block=256, stream=0):
        """One cooperative launch of the replay kernel over nseg epochs separated by
        device-side epoch splits (xpl_grid_epoch); d_seg = nseg+1 event offsets."""
        check("xplw_replay_split", xplw_replay_split(d_addr, d_size, d_acc, d_seg, nseg, grid, block, stream))


def handle_replay(base, elem, d_idx, n, kind, grid=0, block=256, stream=0):
    """Accesses through one array handle of `elem`-byte elements made from `base`:
    element d_idx[i] (int64, any sign) with kind 1 R / 2 W / 3 RW (libxplwork)."""
    if grid <= 0:
        grid = max(1, min((n + block - 1) // block, 148 * 8))
    check("xplw_handle_replay", xplw_handle_replay(base, elem, d_idx, n, kind, grid, block, stream))


def stream_kernel(x_ptr, y_ptr, n, elem, instrumented, stream=0):
    """y[i] = 2 x[i] over n elements of `elem` bytes (4 or 8): the instrumented
    streaming kernel (inside an epoch; instrumented = 1 plain hooks, 2 array
    handles) or its twin (0) (libxplwork.so)."""
    check("xplw_stream", xplw_stream(x_ptr, y_ptr, n, elem, int(instrumented), stream))


def atomic_bench(buf_ptr, n_u32, mode, stream=0):
    """Launch the atomic-throughput microbenchmark kernel (libxplwork): one OR
    per u32 of the device buffer; mode 0 RED, 1 ATOM, 2 same u32 per warp."""
    check("xplw_atomic_bench", xplw_atomic_bench(buf_ptr, n_u32, mode, stream))


def combine_partials(blobs, thr=50, block_words=0, min_run=256):
    """Combine the partials of all ranks (list of byte blobs) into reports (host only)."""
    raw = b"".join(blobs)
    n = len(raw) // C.sizeof(XplPartial)
    arr = (XplPartial * max(n, 1)).from_buffer_copy(raw if n else bytes(C.sizeof(XplPartial)))
    p = XplDiagParams(thr, block_words, min_run)
    cap = max(n, 1)
    out = (XplAllocReport * cap)()
    m = sz(0)
    check("xpl_combine_partials", xpl_combine_partials(arr, n, C.byref(p), out, cap, C.byref(m)))
    return [{f: getattr(out[i], f) for f, _ in REPORT_FIELDS} for i in range(m.value)]


def partials_from_bytes(blob):
    n = len(blob) // C.sizeof(XplPartial)
    arr = (XplPartial * max(n, 1)).from_buffer_copy(blob if n else bytes(C.sizeof(XplPartial)))
    return [arr[i] for i in range(n)]


def format_reports(reports, names=(), csv=False, only_named=False):
    """tracePrint's text (Fig. 4 layout) or CSV for report dicts; names: list of
    (addr, expr) pairs the reports' name_idx refer to."""
    n = len(reports)
    arr = (XplAllocReport * max(n, 1))()
    for i, r in enumerate(reports):
        for f, _ in REPORT_FIELDS:
            setattr(arr[i], f, r[f])
    nm = (XplName * max(len(names), 1))()
    keep = []
    for i, (a, e) in enumerate(names):
        b = e.encode()
        keep.append(b)
        nm[i].addr, nm[i].expr, nm[i].elem_size = a, b, 0
    need = sz(0)
    cap = 4096
    while True:
        buf = C.create_string_buffer(cap)
        st = xpl_format_reports(arr, n, nm if names else None, len(names), int(csv), int(only_named),
                                buf, cap, C.byref(need))
        if st == 1 and need.value > cap:
            cap = need.value
            continue
        check("xpl_format_reports", st)
        return buf.value.decode()

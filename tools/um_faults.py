"""NEXT-4 (optional part): real unified-memory fault / migration counters (CUPTI,
libxplum.so) next to the xpl page view of the same interval (P:L84-90, P:L227,
P:L427).  Runs in a fresh process: the counters are configured before the CUDA
context exists.  Prints one JSON object.

Three allocations, 32 MiB each, three rounds of:
  A (managed): CPU writes every word, GPU increments word 0 of every 4 KiB page,
               CPU reads every word                  -> anti-pattern 1 (alternating)
  B (managed): CPU writes and reads every word only  -> CPU-only managed data
  C (device):  GPU increments word 0 of every 4 KiB page
A diagnose (no reset) and the page view (4 KiB = 1024-word pages) close each run.
"""
import ctypes as C
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
PKG = os.path.join(ROOT, "paper_conf_ipps_pirkelbauerlvl20_b200")


class UmCounts(C.Structure):
    _fields_ = [(f, C.c_uint64) for f in ("htod_bytes", "dtoh_bytes", "dtod_bytes", "cpu_page_faults",
                                          "gpu_page_fault_groups", "thrashing", "throttling", "remote_map",
                                          "records")]


def main():
    um = C.CDLL(os.path.join(PKG, "libxplum.so"))
    um.xpl_um_read.argtypes = [C.c_uint64, C.c_uint64, C.POINTER(UmCounts), C.c_int]
    um.xpl_um_dropped.restype = C.c_uint64
    um.xpl_um_kinds.restype = C.c_uint32
    st = um.xpl_um_enable(0)  # before any CUDA context
    kinds = um.xpl_um_kinds() if st == 0 else 0

    import numpy as np
    import torch
    from paper_conf_ipps_pirkelbauerlvl20_b200 import apps, xpl
    torch.cuda.set_device(0)
    nbytes = 32 << 20
    words = nbytes // 4
    stride = 1024  # one word per 4 KiB page
    w = apps._w
    w.xplw_touch_mem.argtypes = [C.c_void_p, C.c_uint64, C.c_uint64, C.c_int, C.c_void_p]
    A = w.xplw_alloc_managed(nbytes)
    B = w.xplw_alloc_managed(nbytes)
    Cdev = torch.zeros(words, dtype=torch.int32, device="cuda")
    av = np.ctypeslib.as_array((C.c_uint32 * words).from_address(A))
    bv = np.ctypeslib.as_array((C.c_uint32 * words).from_address(B))
    s = torch.cuda.current_stream().cuda_stream
    rng_w = np.zeros(1, dtype=xpl.HOST_ACCESS_DTYPE)

    def host(addr, kind):
        rng_w[0] = (addr, nbytes, kind)
        ctx.record_host_ranges(rng_w)

    names = {1: "htod_bytes", 2: "dtoh_bytes", 3: "cpu_page_faults", 4: "gpu_page_fault_groups", 5: "thrashing",
             6: "throttling", 7: "remote_map", 8: "dtod_bytes"}
    out = {"config": {"bytes_per_alloc": nbytes, "gpu_stride_words": stride, "rounds": 3},
           "um_enable_status": st, "um_available": st == 0,
           "kinds": [v for k, v in names.items() if kinds >> k & 1]}
    with xpl.Context(pool_words=1 << 25) as ctx:
        ctx.bind()
        ctx.register(A, nbytes, 1)
        ctx.register(B, nbytes, 1)
        ctx.register(Cdev.data_ptr(), nbytes, 0)
        torch.cuda.synchronize()
        if st == 0:
            um.xpl_um_read(0, 0, C.byref(UmCounts()), 1)  # drop set-up records
        for it in range(3):
            av[:] = it + 1  # CPU writes A
            host(A, 2)
            bv[:] = it + 1  # CPU writes B
            host(B, 2)
            ctx.kernel_begin(s)
            assert w.xplw_touch_mem(A, words, stride, 1, s) == 0
            assert w.xplw_touch_mem(Cdev.data_ptr(), words, stride, 1, s) == 0
            ctx.kernel_end(s)
            torch.cuda.synchronize()
            out.setdefault("cpu_sums", []).append(int(av.sum(dtype=np.uint64)) + int(bv.sum(dtype=np.uint64)))
            host(A, 1)  # CPU reads A and B
            host(B, 1)
        torch.cuda.synchronize()
        pages = {r["base"]: r for r in ctx.page_summary(1024)}
        diag = {r["base"]: r for r in ctx.diagnose(reset=False)}
    for name, base in (("A_managed_alternating", A), ("B_managed_cpu_only", B), ("C_device", Cdev.data_ptr())):
        cnt = UmCounts()
        if st == 0:
            assert um.xpl_um_read(base, nbytes, C.byref(cnt), 0) == 0
        p, d = pages[base], diag[base]
        out[name] = {"um": {f: getattr(cnt, f) for f, _ in UmCounts._fields_},
                     "pages": {k: p[k] for k in ("pages", "cpu_pages", "gpu_pages", "shared_pages",
                                                 "false_shared_pages", "alternating_pages", "flags")},
                     "diagnose": {k: d[k] for k in ("alternating", "gpu_acc", "any_acc", "flags")}}
    if st == 0:
        tot = UmCounts()
        um.xpl_um_read(0, 0, C.byref(tot), 1)
        out["all_records"] = {f: getattr(tot, f) for f, _ in UmCounts._fields_}
        out["dropped"] = um.xpl_um_dropped()
        um.xpl_um_disable()
    w.xplw_free_managed(A)
    w.xplw_free_managed(B)
    print(json.dumps(out))
    return 0


if __name__ == "__main__":
    sys.exit(main())

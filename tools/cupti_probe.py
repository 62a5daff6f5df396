"""Probe CUPTI unified-memory counter support (order / library variants); one line per step."""
import ctypes as C
import sys

LIBS = {"cuda129": "/usr/local/cuda/targets/x86_64-linux/lib/libcupti.so",
        "torch": "/opt/prime-rl/.venv/lib/python3.12/site-packages/nvidia/cuda_cupti/lib/libcupti.so.12",
        "triton": "/opt/prime-rl/.venv/lib/python3.12/site-packages/triton/backends/nvidia/lib/cupti/libcupti.so"}


class Cfg(C.Structure):
    _fields_ = [("scope", C.c_int), ("kind", C.c_int), ("deviceId", C.c_uint32), ("enable", C.c_uint32)]


REQ = C.CFUNCTYPE(None, C.POINTER(C.POINTER(C.c_uint8)), C.POINTER(C.c_size_t), C.POINTER(C.c_size_t))
CMP = C.CFUNCTYPE(None, C.c_void_p, C.c_uint32, C.POINTER(C.c_uint8), C.c_size_t, C.c_size_t)
bufs = []


def req(b, sz, mx):
    a = (C.c_uint8 * (8 << 20))()
    bufs.append(a)
    b[0] = C.cast(a, C.POINTER(C.c_uint8))
    sz[0] = 8 << 20
    mx[0] = 0


def cmp(ctx, sid, b, sz, valid):
    print("completed", valid, flush=True)


def main(lib, order):
    cupti = C.CDLL(LIBS[lib])
    cuda = C.CDLL("libcuda.so.1")
    v = C.c_uint32()
    cupti.cuptiGetVersion(C.byref(v))
    print(lib, order, "cupti api version", v.value, flush=True)
    print("cuInit", cuda.cuInit(0), flush=True)
    if order == "ctx_first":
        ctx = C.c_void_p()
        print("ctx", cuda.cuDevicePrimaryCtxRetain(C.byref(ctx), 0), cuda.cuCtxSetCurrent(ctx), flush=True)
    rq, cm = REQ(req), CMP(cmp)
    print("register", cupti.cuptiActivityRegisterCallbacks(rq, cm), flush=True)
    cfgs = (Cfg * 4)(*[Cfg(1, k, 0, 1) for k in (1, 2, 3, 4)])
    if order == "enable_first":
        print("enable", cupti.cuptiActivityEnable(25), flush=True)
        print("configure", cupti.cuptiActivityConfigureUnifiedMemoryCounter(cfgs, 4), flush=True)
    else:
        print("configure", cupti.cuptiActivityConfigureUnifiedMemoryCounter(cfgs, 4), flush=True)
        print("enable", cupti.cuptiActivityEnable(25), flush=True)
    print("enable kernel kind (10)", cupti.cuptiActivityEnable(10), flush=True)


if __name__ == "__main__":
    main(sys.argv[1], sys.argv[2])

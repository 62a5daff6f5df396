"""Sharded mode of libxpl.so (world > 1, include/xpl.h) on one GPU:
R processes, one context each, the collectives over a gloo process group
(xpl.TorchComm), the pools mapped into each other with CUDA IPC (same device
here; NVLink peers on a multi-GPU box).  The library itself does everything
sharded: it cuts allocations into pieces, routes every rank's host records to
their owners (all-to-all), records device accesses into remote pools
(atomics into peer-mapped memory), barriers the epoch close, and exchanges and
combines the diagnosis partials.

The logical program is a seeded trace: its host batches are cut into R
contiguous slices (rank r issues slice r -- the logical host stream is the
rank-ordered concatenation), its device events are dealt round-robin to the
ranks' kernels, registrations / frees / copies / diagnoses are collective.
Every rank's reports must equal the oracle's replay of the unsharded trace,
field by field.  Accesses are aligned to their size (reading D36)."""
import os

import numpy as np
import pytest

from xplgen.trace import DEVICE, HOST, MANAGED, R, RW, W

pytestmark = pytest.mark.gpu


def sharded_trace(seed, n_steps=10):
    rng = np.random.default_rng(seed)
    # small allocations (owned whole by one rank) and large ones (cut into pieces)
    words = [37, 1000, 4096, 70_000, 200_003, 65_536, 5, 131_072 + 9]
    ops, allocs, b = [], [], 0x2000_0000
    for i, w in enumerate(words):
        nb = 4 * w - (2 if i % 3 == 1 else 0)
        ops.append(("REG", b, nb, [DEVICE, MANAGED, HOST][i % 3]))
        allocs.append((b, nb))
        b += ((4 * w + 65535) // 65536 + 1) * 65536

    def events(n, sizes=(4, 8)):
        j = rng.integers(0, len(allocs), size=n)
        sz = rng.choice(sizes, size=n).astype(np.uint64)
        nb = np.array([allocs[x][1] for x in j], np.uint64)
        off = (rng.integers(0, 1 << 40, size=n).astype(np.uint64) % np.maximum(nb // sz, 1)) * sz
        addr = np.array([allocs[x][0] for x in j], np.uint64) + off
        return addr, sz.astype(np.uint32)

    for step in range(n_steps):
        a, z = events(6000)
        ops.append(("HB", a, z, rng.integers(1, 4, size=a.size).astype(np.uint8)))
        k = int(rng.integers(0, len(allocs)))
        nbx = allocs[k][1] // 2 if step % 3 else allocs[k][1]
        if step % 2 == 0:
            ops.append(("X", 0, allocs[k][0], 0x7000_0000, nbx))  # H2D
        else:
            ops.append(("X", 1, 0x7000_0000, allocs[k][0], nbx))  # D2H
        ops.append(("KB",))
        a, z = events(30000)
        ops.append(("DB", a, z, rng.integers(1, 4, size=a.size).astype(np.uint8)))
        k = int(rng.integers(0, len(allocs)))  # a dense kernel over a whole allocation (crosses pieces)
        aa = allocs[k][0] + 4 * np.arange(allocs[k][1] // 4, dtype=np.uint64)
        ops.append(("DB", aa, np.full(aa.size, 4, np.uint32), np.full(aa.size, 1 + step % 3, np.uint8)))
        if step % 4 == 1:  # host records inside the open epoch (D20)
            a, z = events(500)
            ops.append(("HB", a, z, rng.integers(1, 4, size=a.size).astype(np.uint8)))
        ops.append(("KE",))
        if step % 3 == 2:
            ops.append(("X", 3, allocs[1][0], allocs[2][0], 4 * 900))  # D2D (own epoch)
        if step == 5:
            ops.append(("FREE", allocs[4][0]))
            ops.append(("REG", allocs[4][0], 4 * 3000, DEVICE))
            allocs[4] = (allocs[4][0], 4 * 3000)
        thr, blk, mr = [(50, 0, 256), (30, 1000, 16), (90, 64, 1), (50, 0, 300)][step % 4]
        ops.append(("DIAG", thr, blk, mr, int(step % 3 != 1), ()))
    ops += [("FREE", x) for x, _ in allocs]
    ops.append(("DIAG", 50, 0, 256, 1, ()))
    return ops


def _rank(rank, world, port, seed, q):
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    import torch
    import torch.distributed as dist
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        torch.cuda.set_device(0)
        from paper_conf_ipps_pirkelbauerlvl20_b200 import xpl
        ops = sharded_trace(seed)
        comm = xpl.TorchComm()
        ctx = xpl.Context(pool_words=1 << 22, comm=comm)
        s = torch.cuda.current_stream().cuda_stream
        got = []
        for op in ops:
            t = op[0]
            if t == "REG":
                ctx.register(op[1], op[2], op[3])
            elif t == "FREE":
                ctx.free(op[1])
            elif t == "KB":
                ctx.kernel_begin(s)
            elif t == "KE":
                ctx.kernel_end(s)
            elif t == "HB":  # slice `rank` of the logical host batch
                parts = np.array_split(np.arange(op[1].size), world)[rank]
                rec = np.zeros(parts.size, dtype=xpl.HOST_ACCESS_DTYPE)
                rec["addr"], rec["size"], rec["kind"] = op[1][parts], op[2][parts], op[3][parts]
                ctx.record_host(rec)
            elif t == "DB":  # dealt round-robin to the ranks' kernels
                m = np.arange(op[1].size) % world == rank
                if m.any():
                    ta = torch.from_numpy(op[1][m].astype(np.uint64).view(np.int64)).cuda()
                    ts = torch.from_numpy(op[2][m].astype(np.uint32).view(np.int32)).cuda()
                    tk = torch.from_numpy(op[3][m].astype(np.uint8)).cuda()
                    ctx.replay(ta.data_ptr(), ts.data_ptr(), tk.data_ptr(), int(m.sum()), stream=s)
                    torch.cuda.current_stream().synchronize()
            elif t == "X":
                ctx.record_copy(op[2], op[3], op[4], op[1])
            elif t == "DIAG":
                got.append(ctx.diagnose(op[1], op[2], op[3], bool(op[4]), op[5]))
            else:
                raise AssertionError(op)
        ctx.close()
        q.put((rank, got))
    except Exception as ex:  # noqa: BLE001
        import traceback
        q.put((rank, "ERR " + repr(ex) + traceback.format_exc()))
    finally:
        dist.destroy_process_group()


@pytest.mark.parametrize("world,seed", [(2, 1), (3, 2), (2, 3)])
def test_sharded_ranks_equal_oracle(world, seed):
    import torch.multiprocessing as mp
    from oracle import run_trace
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = 29600 + 13 * seed + world + os.getpid() % 500
    procs = [ctx.Process(target=_rank, args=(r, world, port, 0x58504C40 + seed, q)) for r in range(world)]
    for p in procs:
        p.start()
    res = dict(q.get(timeout=600) for _ in procs)
    for p in procs:
        p.join(timeout=60)
    for r in range(world):
        assert not isinstance(res[r], str), res[r]
    exp = run_trace(sharded_trace(0x58504C40 + seed))
    for r in range(world):
        got = res[r]
        assert len(got) == len(exp), (r, len(got), len(exp))
        for k, (g, e) in enumerate(zip(got, exp)):
            assert len(g) == len(e), (r, k, len(g), len(e))
            for gr, er in zip(g, e):
                diff = {f: (gr[f], er[f]) for f in er if gr[f] != er[f]}
                assert not diff, f"rank {r} diag {k} row {er['id']}: (gpu, oracle) {diff}"


def test_nccl_comm_single_rank():
    """The NCCL transport of libxpl.so (xpl_comm_nccl_create) on one rank: the
    three collectives through the function pointers the runtime calls."""
    import ctypes as C
    from paper_conf_ipps_pirkelbauerlvl20_b200 import xpl
    comm = xpl.NcclComm(0, 1, 0, lambda b: b)
    try:
        c = comm.p.contents
        src = (C.c_uint8 * 100)(*range(100))
        dst = (C.c_uint8 * 100)()
        assert c.allgather(c.user, src, 100, dst) == 0 and bytes(dst) == bytes(src)
        sb = (C.c_uint64 * 1)(64)
        rb = (C.c_uint64 * 1)(64)
        dst2 = (C.c_uint8 * 64)()
        assert c.alltoallv(c.user, src, sb, dst2, rb) == 0 and bytes(dst2) == bytes(src)[:64]
        assert c.barrier(c.user) == 0
    finally:
        comm.close()


def _lulesh_rank(rank, world, port, s, steps, q):
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    import torch
    import torch.distributed as dist
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        torch.cuda.set_device(0)
        from paper_conf_ipps_pirkelbauerlvl20_b200 import apps, xpl
        from xplgen import lulesh as L
        spec = L.lulesh_spec(s)
        ar = apps.Arena(spec)
        apps.lulesh_prepare(ar, s, L.topology(s, 0x58504C05))
        hc = torch.zeros(1, dtype=torch.int64, device="cuda")
        st = torch.cuda.Stream()
        with xpl.Context(pool_words=1 << 24, max_rows=256, comm=xpl.TorchComm()) as ctx:
            run = apps.Run(ctx, st.cuda_stream, params=(50, 0, 256), rank=rank, world=world)
            apps.lulesh(run, ar, s, steps, hc)
            q.put((rank, run.reports(), int(hc.item())))
    except Exception as ex:  # noqa: BLE001
        import traceback
        q.put((rank, "ERR " + repr(ex) + traceback.format_exc(), 0))
    finally:
        dist.destroy_process_group()


@pytest.mark.parametrize("world,s", [(2, 8), (3, 24)])
def test_sharded_lulesh_equals_one_gpu_and_oracle(world, s):
    """The sharded LULESH-shaped program (each rank its slab of elements and
    nodes, its slice of the host init; rank 0 the domain's host segments) on a
    sharded context: every rank's reports equal the oracle's replay of the
    single-GPU program (all fields but `base`, the piece owners' addresses) --
    the 1-GPU vs N-GPU report identity of SURVEY §8(d) cfg5."""
    import torch
    import torch.multiprocessing as mp
    from oracle import run_trace
    from paper_conf_ipps_pirkelbauerlvl20_b200 import apps, xpl
    from xplgen import lulesh as L
    steps = 3
    # the single-GPU program and its oracle
    spec = L.lulesh_spec(s)
    ar = apps.Arena(spec)
    topo = L.topology(s, 0x58504C05)
    apps.lulesh_prepare(ar, s, topo)
    hc = torch.zeros(1, dtype=torch.int64, device="cuda")
    st = torch.cuda.Stream()
    with xpl.Context(pool_words=1 << 24) as ctx1:
        run = apps.Run(ctx1, st.cuda_stream, params=(50, 0, 256))
        tmps = apps.lulesh(run, ar, s, steps, hc)
        one = run.reports()
    ops, hooks = L.lulesh_trace(ar.addrs, spec, s, steps, topo, (50, 0, 256), tmps)
    exp = run_trace(ops)
    strip = lambda ds: [[{f: v for f, v in r.items() if f != "base"} for r in d] for d in ds]
    assert strip(one) == strip(exp)
    ctxm = mp.get_context("spawn")
    q = ctxm.Queue()
    port = 29800 + s + world + os.getpid() % 500
    procs = [ctxm.Process(target=_lulesh_rank, args=(r, world, port, s, steps, q)) for r in range(world)]
    for p in procs:
        p.start()
    res = {r: (g, h) for r, g, h in (q.get(timeout=600) for _ in procs)}
    for p in procs:
        p.join(timeout=60)
    for r in range(world):
        assert not isinstance(res[r][0], str), res[r][0]
        assert strip(res[r][0]) == strip(exp), f"rank {r}"

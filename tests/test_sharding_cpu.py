"""Multi-rank sharding on CPU (gloo, world size 2): the exchange-and-combine half
of SURVEY §8(e) without a GPU.

Each rank owns one contiguous piece of every logical allocation.  It builds the
partials of its pieces (counters, run-monoid summaries, cut density blocks) from
the oracle's per-word records -- an independent Python restatement of what
xpl_diagnose_partials computes on the GPU -- exchanges them with
torch.distributed.all_gather_object over gloo, and combines them with the
library's xpl_combine_partials (host-only code of libxpl.so).  Every rank must
get exactly the oracle's report of the unsharded allocations.
"""
import ctypes as C
import os
import re

import numpy as np
import pytest
import torch.distributed as dist
import torch.multiprocessing as mp

from xplgen.trace import DEVICE, HOST, MANAGED, R, RW, W, batch

WC, WG, RCC, RGC, RCG, RGG = 4, 8, 16, 32, 64, 128


def make_trace(seed, sizes=(1000, 37, 4096, 5000, 16, 333)):
    rng = np.random.default_rng(seed)
    ops, allocs = [], []
    b = 0x4000_0000
    for i, nw in enumerate(sizes):
        nb = 4 * nw - (i % 2) * 2
        ops.append(("REG", b, nb, [DEVICE, MANAGED, HOST][i % 3]))
        allocs.append((b, nb))
        b += 4 * nw + 4096
    for step in range(8):
        a_idx = rng.integers(0, len(allocs), size=4000)
        w = np.array([rng.integers(0, (allocs[j][1] + 3) // 4) for j in a_idx])
        addr = np.array([allocs[j][0] for j in a_idx], np.uint64) + 4 * w.astype(np.uint64)
        if step % 2 == 0:
            ops.append(batch("HB", addr, 4, rng.integers(1, 4, size=addr.size)))
        else:
            ops += [("KB",), batch("DB", addr, 4, rng.integers(1, 4, size=addr.size)), ("KE",)]
        j = int(rng.integers(0, len(allocs)))  # a long contiguous range: runs across pieces
        ops.append(("X", 0, allocs[j][0], 0x7000_0000, allocs[j][1] // 2))
    return ops, allocs


def runs_summary(flags, min_run):
    """(len, pre, suf, cnt, sum) of a 0/1 array: leading/trailing ones, complete
    inner runs (bounded by zeros inside the range) of length >= min_run."""
    s = "".join("1" if f else "0" for f in flags)
    n = len(s)
    pre = len(s) - len(s.lstrip("1"))
    if pre == n:
        return (n, n, n, 0, 0)
    suf = len(s) - len(s.rstrip("1"))
    inner = s[pre:n - suf]
    lens = [len(m) for m in re.findall("1+", inner) if len(m) >= min_run]
    return (n, pre, suf, len(lens), sum(lens))


def piece_partial(xpl, o, rid, base, nbytes, kind, goff, nwords, lw, thr, B, min_run):
    recs = np.array([o.peek(rid, w) for w in range(goff, goff + nwords)], dtype=np.int64)
    wc, wg, rcc, rgc, rcg, rgg = [(recs & m) != 0 for m in (WC, WG, RCC, RGC, RCG, RGG)]
    cpu = wc | rcc | rgc
    gpu = wg | rcg | rgg
    p = xpl.XplPartial()
    p.logical_id, p.word_offset, p.words, p.logical_words, p.logical_bytes = rid, goff, nwords, lw, nbytes
    p.base, p.kind, p.live, p.name_idx = base, kind, 1, 0xFFFFFFFF
    for k, v in enumerate([wc, wg, rcc, rcg, rgc, rgg, cpu | gpu, gpu, cpu & gpu & (wc | wg)]):
        p.cnt[k] = int(v.sum())
    for dst, fl in ((p.u_run, wc & ~rcg), (p.d_run, rcc)):
        for k, v in enumerate(runs_summary(fl, min_run)):
            dst[k] = v
    p.blk_first = p.blk_last = (1 << 64) - 1
    if B:
        k0, k1 = goff // B, (goff + nwords - 1) // B
        for k in range(k0, k1 + 1):
            lo, hi = k * B, min(k * B + B, lw)
            plo, phi = max(lo, goff), min(hi, goff + nwords)
            g = int(gpu[plo - goff:phi - goff].sum())
            if lo >= goff and hi <= goff + nwords:  # wholly inside: judged here
                if g >= 1 and 100 * g <= thr * (hi - lo):
                    p.low_density_blocks += 1
                    p.low_density_words += hi - lo
            elif k == k0:
                p.blk_first, p.blk_first_g, p.blk_first_s = k, g, phi - plo
            else:
                p.blk_last, p.blk_last_g, p.blk_last_s = k, g, phi - plo
    p.ever_accessed = int((recs & 0xFC).any())
    return p


def _rank(rank, world, port, seed, params, q):
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        from oracle import Oracle
        from paper_conf_ipps_pirkelbauerlvl20_b200 import xpl
        thr, B, min_run = params
        ops, allocs = make_trace(seed)
        o = Oracle()
        for op in ops:
            o.op(op)
        mine = []
        for rid, ((base, nb), op) in enumerate(zip(allocs, ops)):
            lw = (nb + 3) // 4
            chunk = -(-lw // world)
            goff = rank * chunk
            n = max(0, min(lw, goff + chunk) - goff)
            if n:
                mine.append(piece_partial(xpl, o, rid, base, nb, op[3], goff, n, lw, thr, B, min_run))
        blob = b"".join(bytes(memoryview(p).cast("B")) for p in mine)
        blobs = [None] * world
        dist.all_gather_object(blobs, blob)
        got = xpl.combine_partials(blobs, thr, B, min_run)
        exp = o.diag(thr, B, min_run, 1, ())
        for g, e in zip(got, exp):
            diff = {f: (g[f], e[f]) for f in e if g[f] != e[f]}
            assert not diff, (rank, e["id"], diff)
        assert len(got) == len(exp)
        q.put((rank, "ok"))
    except Exception as ex:  # noqa: BLE001
        q.put((rank, repr(ex)))
    finally:
        dist.destroy_process_group()


@pytest.mark.parametrize("seed,params", [(1, (50, 0, 256)), (2, (30, 64, 8)), (3, (90, 1000, 1)),
                                         (4, (50, 7, 3))])
def test_two_rank_combine_matches_unsharded_oracle(seed, params):
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = 29500 + seed * 7 + os.getpid() % 1000
    procs = [ctx.Process(target=_rank, args=(r, 2, port, 0x58504C20 + seed, params, q)) for r in range(2)]
    for p in procs:
        p.start()
    res = dict(q.get(timeout=240) for _ in procs)
    for p in procs:
        p.join(timeout=60)
    assert res == {0: "ok", 1: "ok"}, res


def _comm_rank(rank, world, port, q):
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        from paper_conf_ipps_pirkelbauerlvl20_b200 import xpl
        comm = xpl.TorchComm()
        c = comm.c
        # all-gather: every rank's 13 bytes, in rank order
        src = (C.c_uint8 * 13)(*[(rank * 31 + i) % 256 for i in range(13)])
        dst = (C.c_uint8 * (13 * world))()
        assert c.allgather(c.user, src, 13, dst) == 0
        assert bytes(dst) == b"".join(bytes((r * 31 + i) % 256 for i in range(13)) for r in range(world))
        # all-to-all with uneven sizes: rank r sends (r + q + 1) bytes of value 16 r + q to rank q
        sb = (C.c_uint64 * world)(*[rank + q + 1 for q in range(world)])
        rb = (C.c_uint64 * world)(*[q + rank + 1 for q in range(world)])
        send = b"".join(bytes([16 * rank + q]) * (rank + q + 1) for q in range(world))
        recv = (C.c_uint8 * sum(rb))()
        assert c.alltoallv(c.user, send, sb, recv, rb) == 0
        assert bytes(recv) == b"".join(bytes([16 * q + rank]) * (q + rank + 1) for q in range(world))
        assert c.barrier(c.user) == 0
        q.put((rank, "ok"))
    except Exception as ex:  # noqa: BLE001
        q.put((rank, repr(ex)))
    finally:
        dist.destroy_process_group()


@pytest.mark.parametrize("world", [2, 3])
def test_torch_comm_collectives_gloo(world):
    """The collectives a sharded context calls (xpl.TorchComm, the xpl_comm the
    runtime gets): all-gather and the uneven all-to-all that routes host records
    to their owners, through the same ctypes function pointers libxpl.so calls."""
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = 29700 + world * 11 + os.getpid() % 1000
    procs = [ctx.Process(target=_comm_rank, args=(r, world, port, q)) for r in range(world)]
    for p in procs:
        p.start()
    res = dict(q.get(timeout=240) for _ in procs)
    for p in procs:
        p.join(timeout=60)
    assert res == {r: "ok" for r in range(world)}, res

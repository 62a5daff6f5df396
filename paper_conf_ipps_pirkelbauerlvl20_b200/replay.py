"""Drive an event trace (xplgen.trace format) through the C-ABI.

Host events go to xpl_record_host in program order, transfers to
xpl_record_copy, device events are issued on the GPU by the instrumented
replay kernel of libxplwork.so (each thread calls the xpl_read/xpl_write
hooks), epochs are xpl_kernel_begin/_end around those launches, and DIAG is
xpl_diagnose.  Returns the list of diagnose results (lists of row dicts) --
the same shape as oracle.run_trace, so the tests compare them field by field.
"""
from __future__ import annotations

import numpy as np

from .xpl import HOST_ACCESS_DTYPE, Context


def _host_array(items):
    a = np.zeros(len(items), dtype=HOST_ACCESS_DTYPE)
    if items:
        arr = np.array(items, dtype=np.uint64)
        a["addr"], a["size"], a["kind"] = arr[:, 0], arr[:, 1], arr[:, 2]
    return a


def _group_splits(ops):
    """Fold every maximal chain of >= 2 consecutive top-level epochs
    (KB dev* KE KB dev* KE ...) into one ("SPLIT", [segments]) op: one cooperative
    launch with a device-side epoch split between segments (NEXT-2)."""
    out, i, depth = [], 0, 0
    while i < len(ops):
        if ops[i][0] == "KB" and depth == 0:
            segs, j = [], i
            while j < len(ops) and ops[j][0] == "KB":
                k = j + 1
                while k < len(ops) and ops[k][0] in ("D", "DB"):
                    k += 1
                if k >= len(ops) or ops[k][0] != "KE":
                    break
                segs.append(ops[j + 1:k])
                j = k + 1
            if len(segs) >= 2:
                out.append(("SPLIT", segs))
                i = j
                continue
        if ops[i][0] == "KB":
            depth += 1
        elif ops[i][0] == "KE":
            depth -= 1
        out.append(ops[i])
        i += 1
    return out


def _dev_arrays(evs):
    a, s, k = [], [], []
    for op in evs:
        if op[0] == "D":
            a.append(np.array([op[1]], np.uint64)), s.append(np.array([op[2]], np.uint32))
            k.append(np.array([op[3]], np.uint8))
        else:
            a.append(np.asarray(op[1], np.uint64)), s.append(np.asarray(op[2], np.uint32))
            k.append(np.asarray(op[3], np.uint8))
    if not a:
        return np.zeros(0, np.uint64), np.zeros(0, np.uint32), np.zeros(0, np.uint8)
    return np.concatenate(a), np.concatenate(s), np.concatenate(k)


def run_trace(ops, ctx: Context | None = None, grid=0, block=256, seed=None, host_split=None,
              pool_words=1 << 24, stream=None, split_epochs=False, traced=False, uniform=False):
    """Replay `ops`.  seed: shuffle device events inside every epoch and split
    host batches at random points (metamorphic variants); grid/block: launch
    shape of the replay kernel (grid 0 = enough CTAs for one event each);
    split_epochs: chains of consecutive epochs run as one cooperative launch
    with device-side epoch splits (xpl_grid_epoch) -- must give the same reports;
    traced: device events are launched through the kernel-launch wrapper
    (xpl_trace_kernel_launch, nested into the trace's epoch) -- same reports;
    uniform: an epoch's device events are launched as one K-uniform replay per
    access kind (the compile-time-kind hooks of xpl_read/_write/_rw call sites;
    order inside an epoch does not matter, D5) -- same reports."""
    import torch

    if split_epochs:
        ops = _group_splits(ops)

    rng = np.random.default_rng(seed) if seed is not None else None
    own = ctx is None
    if own:
        n_reg = sum(1 for op in ops if op[0] == "REG")
        ctx = Context(pool_words=pool_words, max_rows=max(4096, n_reg + 16))
    if stream is None:
        stream = torch.cuda.current_stream().cuda_stream
    results = []
    host_items = []
    dev = []  # (addr, size, acc) arrays of the open epoch, launched at flush points

    def flush_host():
        if not host_items:
            return
        arr = _host_array(host_items)
        host_items.clear()
        if rng is not None and host_split and arr.size > 1:
            cuts = np.sort(rng.choice(np.arange(1, arr.size), size=min(host_split, arr.size - 1), replace=False))
            for part in np.split(arr, cuts):
                ctx.record_host(part)
        else:
            ctx.record_host(arr)

    def flush_dev():
        if not dev:
            return
        a = np.concatenate([d[0] for d in dev]).astype(np.uint64)
        s = np.concatenate([d[1] for d in dev]).astype(np.uint32)
        k = np.concatenate([d[2] for d in dev]).astype(np.uint8)
        dev.clear()
        if rng is not None:
            p = rng.permutation(a.size)
            a, s, k = a[p], s[p], k[p]
        if uniform:
            keep = []
            for kind in (1, 2, 3):
                m = k == kind
                if not m.any():
                    continue
                ta = torch.from_numpy(np.ascontiguousarray(a[m]).view(np.int64)).cuda()
                ts = torch.from_numpy(np.ascontiguousarray(s[m]).view(np.int32)).cuda()
                keep += [ta, ts]
                ctx.replay_k(ta.data_ptr(), ts.data_ptr(), int(m.sum()), kind, grid=grid, block=block,
                             stream=stream)
            torch.cuda.current_stream().synchronize()
            return
        ta = torch.from_numpy(a.view(np.int64)).cuda()
        ts = torch.from_numpy(s.view(np.int32)).cuda()
        tk = torch.from_numpy(k).cuda()
        (ctx.replay_traced if traced else ctx.replay)(ta.data_ptr(), ts.data_ptr(), tk.data_ptr(), a.size,
                                                      grid=grid, block=block, stream=stream)
        torch.cuda.current_stream().synchronize()  # keep the temporaries alive until the launch ran

    for op in ops:
        t = op[0]
        if t not in ("H", "HB"):
            flush_host()
        if t == "REG":
            ctx.register(op[1], op[2], op[3])
        elif t == "FREE":
            ctx.free(op[1])
        elif t == "KB":
            flush_dev()
            ctx.kernel_begin(stream)
        elif t == "KE":
            flush_dev()
            ctx.kernel_end(stream)
        elif t == "H":
            host_items.append((op[1], op[2], op[3]))
        elif t == "HB":
            host_items.extend(zip(op[1].tolist(), op[2].tolist(), op[3].tolist()))
        elif t == "D":
            dev.append((np.array([op[1]], np.uint64), np.array([op[2]], np.uint32), np.array([op[3]], np.uint8)))
        elif t == "DB":
            dev.append((np.asarray(op[1], np.uint64), np.asarray(op[2], np.uint32), np.asarray(op[3], np.uint8)))
        elif t == "SPLIT":
            flush_dev()
            parts = [_dev_arrays(seg) for seg in op[1]]
            if rng is not None:
                parts = [tuple(x[p] for x in pt) for pt in parts for p in [rng.permutation(pt[0].size)]]
            off = np.zeros(len(parts) + 1, np.uint64)
            off[1:] = np.cumsum([pt[0].size for pt in parts])
            a = np.concatenate([pt[0] for pt in parts])
            sz = np.concatenate([pt[1] for pt in parts])
            kk = np.concatenate([pt[2] for pt in parts])
            ta = torch.from_numpy(a.view(np.int64)).cuda()
            ts = torch.from_numpy(sz.view(np.int32)).cuda()
            tk = torch.from_numpy(kk).cuda()
            to = torch.from_numpy(off.view(np.int64)).cuda()
            ctx.kernel_begin(stream)
            ctx.replay_split(ta.data_ptr(), ts.data_ptr(), tk.data_ptr(), to.data_ptr(), len(parts),
                             grid=grid, block=block, stream=stream)
            ctx.kernel_end(stream)
            torch.cuda.current_stream().synchronize()
        elif t == "X":
            flush_dev()
            ctx.record_copy(op[2], op[3], op[4], op[1])
        elif t == "PAGES":
            flush_dev()
            results.append(ctx.page_summary(op[1]))
        elif t == "ADVISE":
            ctx.mem_advise(op[1], op[2], op[3], op[4])
        elif t == "DIAG":
            results.append(ctx.diagnose(op[1], op[2], op[3], bool(op[4]), op[5]))
        else:
            raise ValueError(op)
    flush_host()
    if own:
        ctx.close()
    return results

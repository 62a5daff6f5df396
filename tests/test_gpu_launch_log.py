"""NEXT-4: the kernel-launch wrapper and its log (traceKernelLaunch,
P:L227).  Reports through the wrapper stay bit-exact vs the oracle; the log
holds every wrapped launch with its parameters; each epoch's written-chunk count
is bounded by the words it takes over from the CPU (zero iff none) and the
counts add up to the runtime's own fold total; epoch times are positive.  Run
on a B200."""
import numpy as np
import pytest

from oracle import run_trace as oracle_run
from xplgen.trace import random_trace

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def gpu():
    import torch
    assert torch.cuda.is_available(), "GPU tests need a B200 (run under gpurun)"
    from paper_conf_ipps_pirkelbauerlvl20_b200 import replay, xpl
    return replay, xpl


def written_words_per_epoch(ops):
    """Per outermost KB..KE epoch that launches (has device events): the set of
    (alloc id, word) its W / RW events write whose last writer at the epoch's
    start was the CPU (clipped to the allocation; misses ignored) -- the
    words whose pending GPU write the epoch close folds (a word the GPU wrote
    last already ends the epoch GPU-owned, D34).  Test-side bookkeeping of the
    trace (who wrote a word last), no record arithmetic."""
    live, nid, out, depth, cur, has_d, gpu_last = {}, 0, [], 0, None, False, set()

    def words(a, sz):
        for base, (i, nb) in live.items():
            if base <= a < base + nb:
                w0, w1 = (a - base) >> 2, min((nb + 3) // 4 - 1, (a + sz - 1 - base) >> 2)
                return [(i, w) for w in range(w0, w1 + 1)]
        return []

    pending_host = []
    for op in ops:
        t = op[0]
        if t == "REG":
            live[op[1]] = (nid, op[2])
            nid += 1
        elif t == "FREE":
            i = live.pop(op[1])[0]
            gpu_last = {x for x in gpu_last if x[0] != i}
        elif t == "KB":
            if depth == 0:
                cur, has_d = set(), False
            depth += 1
        elif t == "KE":
            depth -= 1
            if depth == 0:
                if has_d:
                    out.append({x for x in cur if x not in gpu_last})
                gpu_last |= cur
                for a, sz in pending_host:  # host writes issued inside the epoch (D20)
                    gpu_last -= set(words(a, sz))
                pending_host = []
        elif t in ("D", "DB"):
            evs = [(op[1], op[2], op[3])] if t == "D" else zip(op[1], op[2], op[3])
            for a, sz, k in evs:
                has_d = True
                if int(k) & 2:
                    cur.update(words(int(a), int(sz)))
        elif t in ("H", "HB"):
            evs = [(op[1], op[2], op[3])] if t == "H" else zip(op[1], op[2], op[3])
            for a, sz, k in evs:
                if int(k) & 2:
                    if depth:
                        pending_host.append((int(a), int(sz)))
                    else:
                        gpu_last -= set(words(int(a), int(sz)))
        elif t == "X":
            assert op[1] in (0, 2), op  # (the test traces drop GPU-side copies)
            gpu_last -= set(words(op[2], op[4]))
    return out


@pytest.mark.parametrize("seed", range(3))
def test_traced_launches_parity_and_log(gpu, seed):
    replay, xpl = gpu
    ops = [o for o in random_trace(0x58504C70 + seed, n_allocs=5, n_steps=90, max_words=6000, p_device=0.8)
           if o[0] != "X"]  # copies make epochs of their own (no launch to log)
    with xpl.Context(pool_words=1 << 22) as ctx:
        ctx.launch_log_enable(True)
        f0 = ctx.stats()["fold_chunks"]
        got = replay.run_trace(ops, ctx=ctx, traced=True, block=128)
        log = ctx.launch_log(reset=True)
        f1 = ctx.stats()["fold_chunks"]
        assert ctx.launch_log() == []
    assert got == oracle_run(ops)
    wsets = written_words_per_epoch(ops)
    epochs = sorted({r["epoch"] for r in log})
    assert len(epochs) == len(wsets) and len(log) >= len(wsets)
    assert [r["seq"] for r in log] == list(range(len(log)))
    for r in log:
        assert r["name"] == "replay_kernel" and r["block"] == (128, 1, 1) and r["shmem"] == 0
        assert r["grid"][1:] == (1, 1) and r["threads"] == r["grid"][0] * 128
        assert r["launches_in_epoch"] == sum(1 for q in log if q["epoch"] == r["epoch"])
        assert r["epoch_ms"] > 0
    chunks = {r["epoch"]: r["epoch_written_chunks"] for r in log}
    total = 0
    for e, ws in zip(epochs, wsets):
        n = len(ws)
        assert (chunks[e] == 0) == (n == 0), (e, chunks[e], n)
        assert -(-n // 128) <= chunks[e] <= n, (e, chunks[e], n)
        total += chunks[e]
    assert total == f1 - f0


def test_launch_log_states(gpu):
    _, xpl = gpu
    import torch
    s = torch.cuda.current_stream().cuda_stream
    with xpl.Context(pool_words=1 << 20) as ctx:
        with pytest.raises(xpl.XplError):  # outside an epoch
            ctx.kernel_launch(s, "k", (1,), (32,))
        ctx.kernel_begin(s)
        ctx.kernel_launch(s, "k", (1,), (32,))  # log off: accepted, not kept
        with pytest.raises(xpl.XplError):  # reading / toggling inside an epoch
            ctx.launch_log()
        with pytest.raises(xpl.XplError):
            ctx.launch_log_enable(True)
        ctx.kernel_end(s)
        assert ctx.launch_log() == []
        ctx.launch_log_enable(True)
        for k in range(3):  # nested begins: one epoch, three launches
            ctx.kernel_begin(s)
        for name in ("a", "b", "a"):
            ctx.kernel_launch(s, name, (2, 3), (4, 5, 6), 7)
        for k in range(3):
            ctx.kernel_end(s)
        log = ctx.launch_log(reset=False)
        assert [r["name"] for r in log] == ["a", "b", "a"] and log[0]["name_idx"] == log[2]["name_idx"]
        assert {r["epoch"] for r in log} == {log[0]["epoch"]} and log[0]["launches_in_epoch"] == 3
        assert log[1]["grid"] == (2, 3, 1) and log[1]["block"] == (4, 5, 6) and log[1]["threads"] == 720
        assert log[1]["shmem"] == 7 and log[0]["epoch_written_chunks"] == 0
        assert len(ctx.launch_log()) == 3 and ctx.launch_log() == []


def test_rodinia_launch_log(gpu):
    """The Rodinia-shaped hotspot logs one launch per iteration with its real
    launch shape; each epoch writes one whole 256 x 300 float grid (76 800
    words: 600 chunks of 128 words, 601 if the row is not chunk-aligned)."""
    _, xpl = gpu
    import torch
    from paper_conf_ipps_pirkelbauerlvl20_b200 import apps
    from xplgen import rodinia
    R, Cc, iters = 256, 300, 4
    spec = rodinia.hotspot_spec(R, Cc)
    ar = apps.Arena(spec)
    rodinia.fill_inputs("hotspot", ar.host_views(), 0x58504C01)
    s = torch.cuda.Stream()
    with xpl.Context(pool_words=1 << 24) as ctx:
        ctx.launch_log_enable(True)
        run = apps.Run(ctx, s.cuda_stream, do_copies=True, diag_each=True)
        apps.hotspot(run, ar, R, Cc, iters)
        log = ctx.launch_log()
    assert [r["name"] for r in log] == ["hotspot_kernel"] * iters
    assert len({r["epoch"] for r in log}) == iters
    for k, r in enumerate(log):
        assert r["grid"] == ((Cc + 31) // 32, (R + 7) // 8, 1) and r["block"] == (32, 8, 1)
        assert r["launches_in_epoch"] == 1 and r["stream"] == s.cuda_stream and r["epoch_ms"] > 0
        # the ping-pong grids are CPU-written (H2D) until the GPU's first write of each:
        # the first two epochs take over 600 chunks each, later ones none (D34)
        if k < 2:
            assert 600 <= r["epoch_written_chunks"] <= 601
        else:
            assert r["epoch_written_chunks"] == 0


def test_launch_log_multi_stream_epoch(gpu):
    """One epoch spanning two streams (D19: begin on s1, a nested begin on s2, the
    outermost end on s1): one epoch entry, both launches in it, its footprint the
    chunks both launches write, reports still bit-exact vs the oracle."""
    replay, xpl = gpu
    import torch
    s1, s2 = torch.cuda.Stream(), torch.cuda.Stream()
    base = 1 << 44
    words = 1 << 16
    with xpl.Context(pool_words=1 << 20) as ctx:
        ctx.register(base, 4 * words, 0)
        ctx.launch_log_enable(True)
        ctx.kernel_begin(s1.cuda_stream)
        ctx.kernel_begin(s2.cuda_stream)
        for st, w0 in ((s1, 0), (s2, 128 * 20)):  # 10 + 10 chunks, disjoint
            addr = torch.arange(base + 4 * w0, base + 4 * (w0 + 128 * 10), 4, dtype=torch.int64, device="cuda")
            sz = torch.full_like(addr, 4, dtype=torch.int32)
            acc = torch.full_like(addr, 2, dtype=torch.uint8)
            torch.cuda.synchronize()
            ctx.kernel_launch(st.cuda_stream, "writer", (addr.numel() // 256,), (256,))
            ctx.replay(addr.data_ptr(), sz.data_ptr(), acc.data_ptr(), addr.numel(), stream=st.cuda_stream)
            torch.cuda.synchronize()
        ctx.kernel_end(s2.cuda_stream)
        ctx.kernel_end(s1.cuda_stream)
        log = ctx.launch_log()
        rep = ctx.diagnose(50, 0, 256, True, ())
    assert [r["stream"] for r in log] == [s1.cuda_stream, s2.cuda_stream]
    assert log[0]["epoch"] == log[1]["epoch"] and log[0]["launches_in_epoch"] == 2
    assert 20 <= log[0]["epoch_written_chunks"] <= 22 and log[0]["epoch_ms"] > 0  # (row start vs chunk grid)
    assert rep[0]["w_g"] == 128 * 20

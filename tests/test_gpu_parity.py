"""GPU parity: the CUDA path, driven through the C-ABI, against the oracle on the
same seeded traces -- element by element, every report field, bit-exact
(all state is integer).  Run on a B200: pytest -m gpu."""
import itertools
import os

import numpy as np
import pytest

from oracle import run_trace as oracle_run
from xplgen.trace import (epoch_chain_trace, DEVICE, MANAGED, RW, SEG_OPS, R, W, enumerated_trace, parse_text, random_trace,
                          schedules)

pytestmark = pytest.mark.gpu

GOLDEN = os.path.join(os.path.dirname(os.path.abspath(__file__)), "golden")


@pytest.fixture(scope="module")
def gpu():
    import torch
    assert torch.cuda.is_available(), "GPU tests need a B200 (run under gpurun)"
    from paper_conf_ipps_pirkelbauerlvl20_b200 import replay, xpl
    return replay, xpl


def compare(got, exp, what=""):
    assert len(got) == len(exp), f"{what}: {len(got)} diagnoses vs {len(exp)}"
    for k, (g, e) in enumerate(zip(got, exp)):
        assert len(g) == len(e), f"{what} diag {k}: {len(g)} rows vs {len(e)}"
        for gr, er in zip(g, e):
            diff = {f: (gr[f], er[f]) for f in er if gr[f] != er[f]}
            assert not diff, f"{what} diag {k} row {er['id']}: (gpu, oracle) {diff}"


@pytest.mark.parametrize("name", sorted(f for f in os.listdir(GOLDEN) if f.endswith(".trace")))
def test_golden(gpu, name):
    replay, _ = gpu
    ops = parse_text(open(os.path.join(GOLDEN, name)).read())
    compare(replay.run_trace(ops), oracle_run(ops), name)


@pytest.mark.parametrize("schedule", schedules(3), ids=lambda s: "".join(s[0]) + "".join("d" if x else "-" for x in s[1]))
def test_bruteforce(gpu, schedule):
    replay, _ = gpu
    nseg = len(schedule[0])
    if nseg <= 2:
        asg = list(itertools.product(SEG_OPS, repeat=nseg))
    else:
        rng = np.random.default_rng(0x58504C00)
        allasg = list(itertools.product(range(len(SEG_OPS)), repeat=3))
        pick = rng.choice(len(allasg), size=20000, replace=False)
        asg = [tuple(SEG_OPS[i] for i in allasg[p]) for p in pick]
    for kind in (MANAGED, DEVICE):
        ops = enumerated_trace(schedule, asg, kind=kind)
        compare(replay.run_trace(ops, pool_words=1 << 26), oracle_run(ops), f"kind={kind}")


@pytest.mark.parametrize("seed", range(24))
def test_random(gpu, seed):
    replay, _ = gpu
    ops = random_trace(0x58504C00 + seed, n_allocs=6, n_steps=80, max_words=5000)
    exp = oracle_run(ops)
    compare(replay.run_trace(ops), exp, "plain")
    # metamorphic: shuffled device events, other launch shapes, split host batches
    compare(replay.run_trace(ops, seed=seed, grid=3, block=64, host_split=5), exp, "shuffled")
    compare(replay.run_trace(ops, seed=seed + 1000, grid=1, block=32, host_split=1), exp, "1 warp")


def big_trace(seed, words=(100_003, 32_768, 65_536 + 17, 1, 16, 31), n_events=400_000):
    """Several tiles per allocation and ragged tails; dense and sparse accesses."""
    rng = np.random.default_rng(seed)
    ops, bases = [], []
    b = 0x2000_0000
    for i, w in enumerate(words):
        ops.append(("REG", b, 4 * w - (i % 3), i % 3))
        bases.append((b, 4 * w - (i % 3)))
        b += ((4 * w + 65535) // 65536 + 1) * 65536
    for epoch in range(6):
        # host segment: a contiguous init of one array + random accesses
        bb, nb = bases[epoch % len(bases)]
        ops.append(("X", 0, bb, 0x7000_0000, nb // 2))
        j = rng.integers(0, len(bases), size=20000)
        off = rng.integers(0, 1 << 30, size=20000) % np.array([n for _, n in bases])[j]
        addr = np.array([bases[x][0] for x in j], dtype=np.uint64) + off.astype(np.uint64)
        ops.append(("HB", addr, rng.choice([1, 4, 8], size=addr.size).astype(np.uint32),
                    rng.integers(1, 4, size=addr.size).astype(np.uint8)))
        ops.append(("KB",))
        j = rng.integers(0, len(bases), size=n_events)
        off = rng.integers(0, 1 << 30, size=n_events) % np.array([n for _, n in bases])[j]
        addr = np.array([bases[x][0] for x in j], dtype=np.uint64) + (off & ~3).astype(np.uint64)
        ops.append(("DB", addr, np.full(addr.size, 4, np.uint32), rng.integers(1, 4, size=addr.size).astype(np.uint8)))
        # a dense streaming kernel over one allocation
        bb, nb = bases[(epoch + 1) % len(bases)]
        a = bb + 4 * np.arange(nb // 4, dtype=np.uint64)
        ops.append(("DB", a, np.full(a.size, 4, np.uint32), np.full(a.size, 1 + epoch % 3, np.uint8)))
        ops.append(("KE",))
        thr, blk, mr = [(50, 0, 256), (30, 1000, 16), (90, 64, 1), (50, 32768, 300), (10, 7, 3), (100, 0, 1)][epoch]
        ops.append(("DIAG", thr, blk, mr, int(epoch % 2 == 0), ()))
        if epoch == 3:
            ops.append(("FREE", bases[0][0]))
            ops.append(("REG", bases[0][0], 4 * 777, 0))
            bases[0] = (bases[0][0], 4 * 777)
    return ops


@pytest.mark.parametrize("seed", range(3))
def test_multi_tile(gpu, seed):
    replay, _ = gpu
    ops = big_trace(0x58504C00 + seed)
    compare(replay.run_trace(ops, pool_words=1 << 24), oracle_run(ops), "big")


def test_small_staging(gpu):
    replay, xpl = gpu
    ops = random_trace(0x58504C77, n_allocs=6, n_steps=60, max_words=5000)
    exp = oracle_run(ops)
    with xpl.Context(pool_words=1 << 22, staging_recs=5) as ctx:
        compare(replay.run_trace(ops, ctx=ctx), exp, "tiny staging")
        st = ctx.stats()
        assert st["folds"] > 0 and st["fold_chunks"] > 0


def test_shadow_dump_matches_oracle(gpu):
    replay, xpl = gpu
    from oracle import Oracle
    ops = random_trace(0x58504C55, n_allocs=4, n_steps=40, max_words=3000)
    ops = [o for o in ops if o[0] != "DIAG"]  # keep the interval bits
    o = Oracle()
    for op in ops:
        o.op(op)
    with xpl.Context(pool_words=1 << 22) as ctx:
        replay.run_trace(ops, ctx=ctx)
        live = {}
        rid = 0
        for op in ops:
            if op[0] == "REG":
                live[op[1]] = (rid, op[2])
                rid += 1
        for base, (rid, nb) in live.items():
            try:
                got = ctx.shadow_dump(base, 0, (nb + 3) // 4)
            except xpl.XplError:
                continue  # freed
            exp = np.array([o.peek(rid, w) for w in range((nb + 3) // 4)], dtype=np.uint8)
            assert np.array_equal(got & 0xFD, exp), base  # bit1 (P) is GPU-internal and 0 here


def test_api_errors(gpu):
    _, xpl = gpu
    import torch
    s = torch.cuda.current_stream().cuda_stream
    with xpl.Context(pool_words=1 << 16, max_rows=4) as ctx:
        assert ctx.diagnose() == []
        ctx.register(0x1000, 64, 1)
        with pytest.raises(xpl.XplError) as e:
            ctx.register(0x1020, 64, 1)
        assert e.value.status == 3
        with pytest.raises(xpl.XplError) as e:
            ctx.free(0x1004)
        assert e.value.status == 4
        with pytest.raises(xpl.XplError) as e:
            ctx.kernel_end(s)
        assert e.value.status == 5
        ctx.kernel_begin(s)
        with pytest.raises(xpl.XplError) as e:
            ctx.diagnose()
        assert e.value.status == 5
        with pytest.raises(xpl.XplError) as e:
            ctx.register(0x9000, 4, 0)
        assert e.value.status == 5
        ctx.kernel_end(s)
        with pytest.raises(xpl.XplError) as e:
            ctx.register(0x5000, 0, 0)
        assert e.value.status == 1
        for i in range(3):
            ctx.register(0x10000 * (i + 2), 8, 0)
        with pytest.raises(xpl.XplError) as e:  # table full
            ctx.register(0x100000, 8, 0)
        assert e.value.status == 2
        with pytest.raises(xpl.XplError) as e:  # pool full
            ctx.free(0x20000)
            ctx.register(0x200000, 4 << 20, 0)
        assert e.value.status == 2


@pytest.mark.parametrize("seed", range(6))
def test_host_ranges(gpu, seed):
    """xpl_record_host_ranges: byte ranges that may span several allocations and
    the gaps between them == the same bytes as one-byte host accesses."""
    replay, xpl = gpu
    import torch
    rng = np.random.default_rng(0x58504C10 + seed)
    ops = []
    bases = []
    b = 0x3000_0000
    for i in range(8):
        n = int(rng.integers(1, 200))
        ops.append(("REG", b, n, i % 3))
        bases.append((b, n))
        b += n + int(rng.integers(0, 3)) * 4  # adjacent allocations and small gaps
    lo, hi = bases[0][0] - 16, b + 16
    ranges = []
    for _ in range(300):
        a = int(rng.integers(lo, hi))
        n = int(rng.integers(1, 64))
        ranges.append((a, n, int(rng.integers(1, 3))))  # R or W (RW runs need word alignment)
    # oracle: every byte as its own access, in order
    for a, n, k in ranges:
        ops.append(("HB", np.arange(a, a + n, dtype=np.uint64), np.ones(n, np.uint32), np.full(n, k, np.uint8)))
    ops.append(("DIAG", 50, 0, 1, 1, ()))
    exp = oracle_run(ops)
    with xpl.Context(pool_words=1 << 20) as ctx:
        for op in ops[:8]:
            ctx.register(op[1], op[2], op[3])
        rec = np.zeros(len(ranges), dtype=xpl.HOST_ACCESS_DTYPE)
        rec["addr"] = [r[0] for r in ranges]
        rec["size"] = [r[1] for r in ranges]
        rec["kind"] = [r[2] for r in ranges]
        ctx.record_host_ranges(rec)
        got = [ctx.diagnose(50, 0, 1, True)]
    compare(got, exp, "ranges")


@pytest.mark.parametrize("seed", [0, 1, 2])
def test_host_strided(gpu, seed):
    """xpl_record_host_strided: strided sequences (positive, negative and zero
    strides; elements in one allocation, spanning several, or untracked;
    some recorded inside an open GPU epoch, so deferred) == every element as
    its own one-byte-per-byte host access, in order."""
    replay, xpl = gpu
    import torch
    rng = np.random.default_rng(0x58504C20 + seed)
    ops, bases = [], []
    b = 0x3100_0000
    for i in range(6):
        n = int(rng.integers(64, 4000))
        ops.append(("REG", b, n, i % 3))
        bases.append((b, n))
        b += n + int(rng.integers(0, 3)) * 4
    lo, hi = bases[0][0] - 64, b + 64
    recs, expanded = [], []
    for _ in range(200):
        size = int(rng.choice([1, 2, 4, 8, 12]))
        kind = int(rng.integers(1, 4))
        if kind == 3:
            size = 4 * int(rng.integers(1, 3))
        stride = int(rng.choice([0, 4, 8, 16, 64, -4, -64, 100, 4 * int(rng.integers(1, 300))]))
        count = int(rng.integers(1, 80))
        a = int(rng.integers(lo, hi))
        if kind == 3:
            a &= ~3
        recs.append((a, size, kind, stride, count))
        expanded += [(a + j * stride, size, kind) for j in range(count)]
    split = len(recs) // 2  # the second half inside a GPU epoch (D20: applied at its close)
    n_first = sum(r[4] for r in recs[:split])

    def host_ops(part):
        out = []
        for a, n, k in part:
            if k == 3:  # RW of a word-aligned range: per word R then W (one access per word)
                out.append(("HB", np.arange(a, a + n, 4, dtype=np.uint64), np.full(n // 4, 4, np.uint32),
                            np.full(n // 4, 3, np.uint8)))
            else:
                out.append(("HB", np.arange(a, a + n, dtype=np.uint64), np.ones(n, np.uint32), np.full(n, k, np.uint8)))
        return out

    ops += host_ops(expanded[:n_first]) + [("KB",)] + host_ops(expanded[n_first:]) + [("KE",)]
    ops.append(("DIAG", 50, 0, 1, 1, ()))
    exp = oracle_run(ops)
    with xpl.Context(pool_words=1 << 20) as ctx:
        for op in ops[:6]:
            ctx.register(op[1], op[2], op[3])
        rec = np.zeros(len(recs), dtype=xpl.HOST_STRIDED_DTYPE)
        for f, k in zip(("addr", "size", "kind", "stride", "count"), range(5)):
            rec[f] = [r[k] for r in recs]
        ctx.record_host_strided(rec[:split])
        s = torch.cuda.current_stream().cuda_stream
        ctx.kernel_begin(s)
        ctx.record_host_strided(rec[split:])
        ctx.kernel_end(s)
        got = [ctx.diagnose(50, 0, 1, True)]
    compare(got, exp, "strided")


def stretch_trace(seed, words=(300_000, 70_001, 16_384 * 3)):
    """Long stretches of identical record bytes (the diagnose kernel's uniform
    512-word fast path) with ragged, unaligned stretch ends, so steps are uniform,
    mixed, and uniform with a different byte than the step before; every access
    recipe is applied to a whole stretch (transfers + dense device batches)."""
    rng = np.random.default_rng(seed)
    ops, allocs = [], []
    b = 0x3000_0000
    for i, w in enumerate(words):
        ops.append(("REG", b, 4 * w, (DEVICE, MANAGED, DEVICE)[i]))
        allocs.append((b, w))
        b += ((4 * w + 65535) // 65536 + 1) * 65536
    recipes = ["HW", "GR", "HR", "GW", "GRW", "HW GR", "GW HR", "HW HR GR GW", "GR HW", ""]
    for rnd in range(3):
        for base, w in allocs:
            cuts = np.sort(rng.choice(np.arange(1, w), size=min(w - 1, 40), replace=False))
            cuts = np.concatenate([[0], cuts, [w]])
            # bias some cuts onto 512-word boundaries
            cuts = np.where(rng.random(cuts.size) < 0.5, (cuts // 512) * 512, cuts)
            cuts = np.unique(np.clip(cuts, 0, w))
            for s, e in zip(cuts[:-1], cuts[1:]):
                if e <= s:
                    continue
                a0, nb = base + 4 * int(s), 4 * int(e - s)
                for step in recipes[int(rng.integers(0, len(recipes)))].split():
                    if step == "HW":
                        ops.append(("X", 0, a0, 0x7000_0000, nb))
                    elif step == "HR":
                        ops.append(("X", 1, 0x7000_0000, a0, nb))
                    else:
                        acc = {"GR": R, "GW": W, "GRW": RW}[step]
                        a = a0 + 4 * np.arange(nb // 4, dtype=np.uint64)
                        ops += [("KB",), ("DB", a, np.full(a.size, 4, np.uint32), np.full(a.size, acc, np.uint8)), ("KE",)]
        for params, reset in (((50, 0, 256), 0), ((50, 0, 1), 0), ((30, 0, 5000), rnd % 2)):
            ops.append(("DIAG", *params, reset, ()))
    return ops


@pytest.mark.parametrize("seed", range(3))
def test_uniform_stretches(gpu, seed):
    replay, _ = gpu
    ops = stretch_trace(0x58504C40 + seed)
    compare(replay.run_trace(ops, pool_words=1 << 22), oracle_run(ops), "stretches")


@pytest.mark.parametrize("tile", ["2048", "4096", "16384", "2048u"])
def test_tile_size_invariance(gpu, tile, monkeypatch):
    """The diagnose kernel's tile size (chosen per call from the call's size) must
    not change any report: the stretch and multi-tile traces under a forced tile
    size equal the oracle (which has no tiles)."""
    replay, _ = gpu
    if tile.endswith("u"):  # the separate stitch kernels (not fused into the tile kernel)
        tile = tile[:-1]
        monkeypatch.setenv("XPL_DIAG_UNFUSED", "1")
    monkeypatch.setenv("XPL_DIAG_TILE_WORDS", tile)
    for ops in (stretch_trace(0x58504C50), big_trace(0x58504C51)):
        compare(replay.run_trace(ops, pool_words=1 << 24), oracle_run(ops), f"tile={tile}")


def long_row_trace(seed, words=(5_000_003, 700_001, 3)):
    """Rows of hundreds to thousands of tiles (the diagnose stitch's two levels:
    segments of 128 tiles, then the row), sparse scattered GPU events, host
    ranges and transfers cut at random words, runs crossing tile and segment
    boundaries; three diagnose parameter sets, with and without reset."""
    rng = np.random.default_rng(seed)
    ops, allocs = [], []
    b = 0x4000_0000
    for i, w in enumerate(words):
        ops.append(("REG", b, 4 * w - (i % 2), (MANAGED, DEVICE, MANAGED)[i]))
        allocs.append((b, w))
        b += ((4 * w + 65535) // 65536 + 1) * 65536
    for rnd in range(3):
        for base, w in allocs:
            s = int(rng.integers(0, w))
            e = min(w, s + int(rng.integers(1, 1 << 21)))
            ops.append(("X", 0, base + 4 * s, 0x7000_0000, 4 * (e - s)))  # H2D of a stretch
        ops.append(("KB",))
        for base, w in allocs:
            n = int(min(w, 60_000))
            a = base + 4 * np.sort(rng.integers(0, w, size=n)).astype(np.uint64)
            ops.append(("DB", a, np.full(n, 4, np.uint32), rng.integers(1, 4, size=n).astype(np.uint8)))
        ops.append(("KE",))
        base, w = allocs[rnd % len(allocs)]
        s = int(rng.integers(0, w))
        ops.append(("X", 1, 0x7000_0000, base + 4 * s, 4 * min(w - s, 300_000)))  # D2H
        for params, reset in (((50, 0, 256), 0), ((50, 0, 1), rnd % 2), ((10, 0, 70_000), 0)):
            ops.append(("DIAG", *params, reset, ()))
    return ops


_EXPECTED = {}


@pytest.mark.parametrize("n", [1, 1023, 8191, 8192, 8193])
def test_merge_segment_sizes(gpu, n):
    """Host segments of exactly n staged records around the single-CTA merge's
    limit (8192 records): scattered non-abutting accesses of every kind, mixed
    with ranges of up to 256 words (a piece's 65 shadow u32s), read before and
    after writes of the same words; device epochs in between so L differs."""
    replay, _ = gpu
    rng = np.random.default_rng(0x58504C70 + n)
    w = 40_000
    base = 0x5000_0000
    ops = [("REG", base, 4 * w, MANAGED), ("KB",),
           ("DB", base + 4 * np.arange(0, w, 3, dtype=np.uint64), np.full(len(range(0, w, 3)), 4, np.uint32),
            np.full(len(range(0, w, 3)), W, np.uint8)), ("KE",)]
    for _ in range(2):
        words = np.sort(rng.choice(w // 2, size=n, replace=False)) * 2  # (never abutting: no coalescing)
        size = np.where(rng.random(n) < 0.05, 4 * rng.integers(2, 257, size=n), 4).astype(np.uint32)
        words = np.minimum(words, w - size // 4)
        perm = rng.permutation(n)
        ops.append(("HB", base + 4 * words[perm].astype(np.uint64), size[perm],
                    rng.integers(1, 4, size=n).astype(np.uint8)))
        ops += [("KB",), ("DB", base + 4 * rng.integers(0, w, size=5000).astype(np.uint64),
                          np.full(5000, 4, np.uint32), rng.integers(1, 4, size=5000).astype(np.uint8)), ("KE",)]
        ops.append(("DIAG", 50, 0, 1, 0, ()))
    compare(replay.run_trace(ops, pool_words=1 << 20), oracle_run(ops), f"n={n}")


@pytest.mark.parametrize("mode", ["fused", "unfused"])
@pytest.mark.parametrize("tile", ["2048", "16384"])
def test_diag_long_rows(gpu, mode, tile, monkeypatch):
    """The diagnose stitch over rows of up to 2442 tiles (20 segments): the fused
    one-launch path (last-warp-done segment and row combines inside the tile
    kernel) and the separate stitch kernels (XPL_DIAG_UNFUSED) both equal the
    oracle, under two forced tile sizes."""
    replay, _ = gpu
    monkeypatch.setenv("XPL_DIAG_TILE_WORDS", tile)
    if mode == "unfused":
        monkeypatch.setenv("XPL_DIAG_UNFUSED", "1")
    ops = long_row_trace(0x58504C60)
    if "long_row" not in _EXPECTED:  # (the oracle takes ~10 s here: once per module)
        _EXPECTED["long_row"] = oracle_run(ops)
    compare(replay.run_trace(ops, pool_words=1 << 23), _EXPECTED["long_row"], f"{mode} tile={tile}")


@pytest.mark.parametrize("seed", range(6))
@pytest.mark.parametrize("grid,block", [(1, 128), (0, 256), (3, 96)])
def test_device_epoch_split(gpu, seed, grid, block):
    """NEXT-2: chains of epochs replayed as ONE cooperative launch with a
    device-side epoch split (xpl_grid_epoch) between them give the oracle's
    reports (= one launch per epoch), for one CTA, the full co-resident grid
    and odd shapes, with the events of each segment shuffled."""
    replay, _ = gpu
    ops = epoch_chain_trace(0x58504C20 + seed)
    exp = oracle_run(ops)
    assert replay.run_trace(ops, grid=grid, block=block, seed=seed, split_epochs=True) == exp


def test_device_epoch_split_random_traces(gpu):
    replay, _ = gpu
    for seed in range(4):
        ops = random_trace(0x58504C30 + seed, n_allocs=5, n_steps=80, max_words=4000, p_device=0.9)
        assert replay.run_trace(ops, split_epochs=True) == oracle_run(ops)


@pytest.mark.parametrize("seed", range(4))
def test_page_view(gpu, seed):
    """NEXT-3: the UM page view (xpl_page_summary, page sizes 1, 5, 16, 1024, huge)
    and recorded cudaMemAdvise hints, bit-exact vs the oracle on random traces."""
    replay, _ = gpu
    from xplgen.trace import with_pages
    ops = with_pages(random_trace(0x58504C60 + seed, n_allocs=6, n_steps=80, max_words=5000),
                      (1, 5, 16, 256, 512, 1024, 1 << 40), seed)
    compare(replay.run_trace(ops), oracle_run(ops), f"pages seed {seed}")


def test_page_flags_map(gpu):
    """xpl_page_flags: the per-page bits of one allocation equal the OR of the
    per-word classes of its shadow dump (pages of 1000 words, ragged tail)."""
    _, xpl = gpu
    ops = random_trace(0x58504C66, n_allocs=3, n_steps=60, max_words=20000, p_device=0.9)
    ops = [o for o in ops if o[0] != "DIAG"]
    from paper_conf_ipps_pirkelbauerlvl20_b200 import replay
    with xpl.Context(pool_words=1 << 22) as ctx:
        replay.run_trace(ops, ctx=ctx)
        for r in ctx.page_summary(1000):
            f = ctx.page_flags(r["base"], 1000, r["pages"])
            d = ctx.shadow_dump(r["base"], 0, r["words"])
            for p in range(r["pages"]):
                w = d[p * 1000:(p + 1) * 1000].astype(np.uint32)
                cpu, gp = (w & 0x34) != 0, (w & 0xC8) != 0
                e = (int(cpu.any()) | 2 * int(gp.any()) | 4 * int((cpu & gp).any()) |
                     8 * int((cpu & gp & ((w & 0x0C) != 0)).any()) | 16 * int(((w & 4) != 0).any()) |
                     32 * int(((w & 8) != 0).any()))
                assert f[p] == e, (r["id"], p)


@pytest.mark.parametrize("seed", range(3))
def test_read_lat_deferred_commit(gpu, seed):
    """xpl_read_lat (the read hook whose commit runs at the end of the full
    expression) gives the records xpl_read gives: device reads of 1, 2, 4, 8 and
    16 bytes (sub-word, one word, multi-word), hits and misses, after random host
    writes, bit-exact vs the oracle through several epochs and diagnoses."""
    _, xpl = gpu
    import torch
    rng = np.random.default_rng(0x58504C80 + seed)
    allocs = [(0x10000000 + k * 0x100000, int(rng.integers(100, 5000)) * 4 + int(rng.integers(0, 4)))
              for k in range(4)]
    ops = [("REG", a, b, int(rng.integers(0, 3))) for a, b in allocs]
    for e in range(10):
        for _ in range(6):
            a, b = allocs[int(rng.integers(4))]
            ops.append(("H", a + int(rng.integers(0, b)), int(rng.integers(1, 64)), int(rng.integers(1, 4))))
        sz = (1, 2, 4, 8, 16)[e % 5]
        n = int(rng.integers(1, 3000))
        picks = rng.integers(0, 4, n)
        addrs = np.array([allocs[p][0] + int(rng.integers(0, allocs[p][1] + 64)) // sz * sz for p in picks],
                         dtype=np.uint64)  # (+64: some reads miss past the end)
        ops += [("KB",), ("DB", addrs, np.full(n, sz, np.uint32), np.full(n, R, np.uint8)), ("KE",),
                ("DIAG", 50, 0, 256, int(e % 3 != 0), ())]
    s = torch.cuda.current_stream().cuda_stream
    got = []
    with xpl.Context(pool_words=1 << 22) as ctx:
        for op in ops:
            t = op[0]
            if t == "REG":
                ctx.register(op[1], op[2], op[3])
            elif t == "H":
                ctx.record_host(np.array([(op[1], op[2], op[3])], dtype=xpl.HOST_ACCESS_DTYPE))
            elif t == "KB":
                ctx.kernel_begin(s)
            elif t == "KE":
                ctx.kernel_end(s)
            elif t == "DB":
                d = torch.from_numpy(op[1].view(np.int64)).cuda()
                grid = int(rng.integers(1, 64))
                xpl.check("xplw_read_lat", xpl.xplw_read_lat(d.data_ptr(), d.numel(), int(op[2][0]), grid, 96, s))
                torch.cuda.synchronize()
            elif t == "DIAG":
                got.append(ctx.diagnose(*op[1:5], names=op[5]))
    compare(got, oracle_run(ops), f"read_lat seed {seed}")

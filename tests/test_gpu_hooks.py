"""GPU parity of the device-hook paths (xpl_device.cuh) against
the oracle: every warp-level case the hooks distinguish, with compile-time
access kinds (the xpl_read / xpl_write / xpl_rw call sites) and per-lane kinds:

  contiguous warps   lane l at words G + l*w: 1-, 2-, 4-, 8-byte elements,
                     aligned and unaligned allocation bases and offsets;
  one address        every lane on the same word / same shadow u32;
  generic            strided, reversed, interleaved, random gathers, partial
                     warps (ragged n, odd block sizes), accesses spanning u32s;
  streaming kernel   the bench's instrumented y[i] = 2 x[i] over a ragged n.

The shadow's last-writer bits differ inside single shadow u32s (host writes of
every other word before the GPU epochs), so the per-byte read classification
(C>G vs G>G) is exercised in every case.  Reports are compared field by field."""
import numpy as np
import pytest

from oracle import run_trace as oracle_run
from xplgen.trace import DEVICE, MANAGED, RW, R, W

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def gpu():
    import torch
    assert torch.cuda.is_available()
    from paper_conf_ipps_pirkelbauerlvl20_b200 import replay, xpl
    return torch, replay, xpl


def compare(got, exp, what=""):
    assert len(got) == len(exp), f"{what}: {len(got)} diagnoses vs {len(exp)}"
    for k, (g, e) in enumerate(zip(got, exp)):
        assert len(g) == len(e), f"{what} diag {k}"
        for gr, er in zip(g, e):
            diff = {f: (gr[f], er[f]) for f in er if gr[f] != er[f]}
            assert not diff, f"{what} diag {k} row {er['id']}: (gpu, oracle) {diff}"


def _u64(x):
    return np.asarray(x, dtype=np.uint64)


def patterns(base, nbytes, rng):
    """(name, addrs, size) device-access patterns inside [base, base+nbytes)."""
    out = []
    for sz in (1, 2, 4, 8, 16):
        n = max(1, min(nbytes // sz, 5000))
        for off in (0, 2, 4, 6) if sz >= 4 else (0, 1):
            m = (nbytes - off) // sz
            if m <= 0:
                continue
            k = min(n, m)
            out.append((f"contig{sz}+{off}", base + off + sz * _u64(np.arange(k)), sz))
        out.append((f"reversed{sz}", base + sz * _u64(np.arange(min(n, nbytes // sz))[::-1]), sz))
        out.append((f"stride2_{sz}", base + 2 * sz * _u64(np.arange(min(n, nbytes // (2 * sz)))), sz))
        out.append((f"random{sz}", base + _u64(rng.integers(0, max(1, nbytes - sz), size=min(n, 3000))), sz))
    out.append(("same_word", _u64(np.full(777, base + 8)), 4))
    out.append(("same_u32_bytes", base + 4 + _u64(np.tile(np.arange(4), 300)), 1))
    out.append(("interleaved", base + 4 * _u64((np.arange(4096) * 5) % 997), 4))
    out.append(("pairs", base + 4 * _u64(np.repeat(np.arange(1500), 2)), 4))
    return out


def hook_trace(seed, kind_mode, alloc_kind):
    """kind_mode: 'uniform' (one kind per epoch) or 'mixed' (per event)."""
    rng = np.random.default_rng(seed)
    sizes = [40_001, 4096, 130, 7]
    ops, bases, b = [], [], 0x3000_0000
    for i, nb in enumerate(sizes):
        base = b + (i % 3)  # unaligned bases too (words count from the base, D2)
        ops.append(("REG", base, nb, alloc_kind))
        bases.append((base, nb))
        b += ((nb + 65535) // 65536 + 1) * 65536
    for e, (base, nb) in enumerate(bases * 2):
        # host writes of every other word: last writers differ inside shadow u32s
        w = base + 8 * _u64(np.arange(nb // 8))
        ops.append(("HB", w, np.full(w.size, 4, np.uint32), np.full(w.size, W, np.uint8)))
        for name, addrs, sz in patterns(base, nb, rng):
            ops.append(("KB",))
            if kind_mode == "uniform":
                kinds = np.full(addrs.size, [R, W, RW][rng.integers(0, 3)], np.uint8)
            else:
                kinds = rng.integers(1, 4, size=addrs.size).astype(np.uint8)
            ops.append(("DB", addrs, np.full(addrs.size, sz, np.uint32), kinds))
            ops.append(("KE",))
        ops.append(("DIAG", 50, 1000 if e % 2 else 0, 3, int(e % 3 != 2), ()))
    return ops


@pytest.mark.parametrize("seed", range(3))
@pytest.mark.parametrize("alloc_kind", [DEVICE, MANAGED])
def test_hook_paths_uniform(gpu, seed, alloc_kind):
    torch, replay, xpl = gpu
    ops = hook_trace(0x58504C10 + seed, "uniform", alloc_kind)
    exp = oracle_run(ops)
    compare(replay.run_trace(ops, uniform=True), exp, "uniform")
    compare(replay.run_trace(ops, uniform=True, block=96, grid=5), exp, "uniform 96x5")
    compare(replay.run_trace(ops, uniform=True, block=33, grid=7, seed=seed), exp, "uniform shuffled 33x7")


@pytest.mark.parametrize("seed", range(3))
def test_hook_paths_mixed(gpu, seed):
    torch, replay, xpl = gpu
    ops = hook_trace(0x58504C20 + seed, "mixed", MANAGED)
    exp = oracle_run(ops)
    compare(replay.run_trace(ops), exp, "per-lane kinds")
    compare(replay.run_trace(ops, uniform=True), exp, "split by kind")
    compare(replay.run_trace(ops, block=64, grid=3, seed=seed), exp, "per-lane kinds shuffled")


@pytest.mark.parametrize("seed", range(8))
def test_random_traces_uniform_kind_launches(gpu, seed):
    torch, replay, xpl = gpu
    from xplgen.trace import random_trace
    ops = random_trace(0x58504C30 + seed, n_allocs=6, n_steps=80, max_words=5000)
    exp = oracle_run(ops)
    compare(replay.run_trace(ops, uniform=True), exp, "uniform")
    compare(replay.run_trace(ops, uniform=True, grid=2, block=160, seed=seed), exp, "uniform shuffled")


@pytest.mark.parametrize("mode", [1, 2])  # plain hooks / array handles
@pytest.mark.parametrize("elem,n", [(4, 1000003), (8, 777777), (4, 31), (8, 1)])
def test_stream_kernel(gpu, elem, n, mode):
    torch, replay, xpl = gpu
    x = torch.arange(n * elem // 4, dtype=torch.int32, device="cuda")
    y = torch.zeros_like(x)
    s = torch.cuda.current_stream().cuda_stream
    xa, ya = x.data_ptr(), y.data_ptr()
    with xpl.Context(pool_words=1 << 24) as ctx:
        ctx.register(xa, n * elem, DEVICE)
        ctx.register(ya, n * elem, DEVICE)
        ctx.record_copy(xa, 0x1000, n * elem // 2, 0)  # H2D of the first half of x
        got = []
        for rep in range(2):  # second epoch: every bit already set (re-touch)
            ctx.kernel_begin(s)
            xpl.stream_kernel(xa, ya, n, elem, mode, s)
            ctx.kernel_end(s)
        got.append(ctx.diagnose(50, 0, 256, reset=True))
        ctx.kernel_begin(s)
        xpl.stream_kernel(xa, ya, n, elem, mode, s)
        ctx.kernel_end(s)
        got.append(ctx.diagnose(50, 0, 256, reset=True))
    torch.cuda.synchronize()
    assert torch.equal(y, (x.view(torch.int64) * 2).view(torch.int32) if elem == 8 else x * 2)
    ia = xa + elem * np.arange(n, dtype=np.uint64)
    ib = ya + elem * np.arange(n, dtype=np.uint64)
    ev = ("DB", np.concatenate([ia, ib]), np.full(2 * n, elem, np.uint32),
          np.concatenate([np.full(n, R, np.uint8), np.full(n, W, np.uint8)]))
    ops = [("REG", xa, n * elem, DEVICE), ("REG", ya, n * elem, DEVICE), ("X", 0, xa, 0x1000, n * elem // 2),
           ("KB",), ev, ("KE",), ("KB",), ev, ("KE",), ("DIAG", 50, 0, 256, 1, ()),
           ("KB",), ev, ("KE",), ("DIAG", 50, 0, 256, 1, ())]
    compare(got, oracle_run(ops), "stream")


@pytest.mark.parametrize("elem", [4, 8, 12])
@pytest.mark.parametrize("shift", [0, 4, 2])
def test_array_handles(gpu, elem, shift):
    """xpl_array handles (the hoisted lookup): a handle made `shift` bytes into
    an allocation (word-aligned or not), elements inside the row, past its end
    (into the next allocation and into untracked memory), before its start
    (negative indices) and straddling the row end -- each event recorded exactly
    as the same access through xpl_read / xpl_write / xpl_rw."""
    torch, replay, xpl = gpu
    rng = np.random.default_rng(elem * 10 + shift)
    a, b = 0x6000_0000, 0x6000_0000 + 4 * 1003 + 2  # b starts right after a's last (partial) word
    na, nb = 4 * 1003 + 2, 4 * 500
    base = a + shift
    nel = (na - shift) // elem
    ops = [("REG", a, na, MANAGED), ("REG", b, nb, MANAGED)]
    with xpl.Context(pool_words=1 << 20) as ctx:
        ctx.register(a, na, MANAGED)
        ctx.register(b, nb, MANAGED)
        s = torch.cuda.current_stream().cuda_stream
        got = []
        for ep in range(4):
            idx = np.concatenate([np.arange(nel), rng.integers(-50, nel + 300, size=3000),
                                  np.array([nel, nel - 1, -1, nel + 200])]).astype(np.int64)
            if ep % 2:
                idx = rng.permutation(idx)
            kind = [1, 2, 3, 1][ep]
            d = torch.from_numpy(idx).cuda()
            ctx.kernel_begin(s)
            xpl.handle_replay(base, elem, d.data_ptr(), idx.size, kind, stream=s)
            ctx.kernel_end(s)
            torch.cuda.synchronize()
            addrs = (base + elem * idx).astype(np.uint64)
            ops += [("KB",), ("DB", addrs, np.full(idx.size, elem, np.uint32), np.full(idx.size, kind, np.uint8)),
                    ("KE",)]
            if ep % 2:
                got.append(ctx.diagnose(50, 0, 16, reset=True))
                ops.append(("DIAG", 50, 0, 16, 1, ()))
    compare(got, oracle_run(ops), "handles")

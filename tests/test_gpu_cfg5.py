"""cfg5 (BASELINE.json configs[4]): the LULESH-shaped program at size 250^3
(15.6 M elements, 15.8 M nodes, 1.47e9 shadow words of persistent arrays plus
0.84e9 of temporaries per timestep) at full size on one B200, two timesteps,
in the program's own launch configuration.

The full event trace (~8e9 accesses per timestep) is far beyond the oracle, so
parity is checked on sampled outputs the oracle can compute one by one
(SURVEY §8(d) cfg5):
  * the complete rows of `dom` (the Fig. 4 object, read by every thread of
    every kernel) and `dt_block` in every diagnose, against the oracle replaying
    the sampled twin (xplgen.lulesh, windows=...), which carries every event of
    those two allocations;
  * per-word records of 8 windows in each of the 48 domain arrays (first,
    ragged last, 6 random), against the oracle's records of the same words
    (a word's record depends only on the events that touch it);
  * and, as a property at any size, every array's counters in the last report
    equal the popcounts of its full shadow dump (D21).
Diagnoses do not reset here (D25: reset = 0 changes nothing else), so the
interval bits of both timesteps stay in the shadow for the dumps.
"""
import numpy as np
import pytest

pytestmark = [pytest.mark.gpu, pytest.mark.slow]

S, STEPS, PARAMS = 250, 2, (50, 0, 256)


def _windows(s, rng):
    from xplgen import lulesh as L
    win = {}
    for k in range(48):
        words = L.slot_bytes(s, k) // 4
        ws = [(0, 1024), (words - 1000, words)]
        for r in rng.integers(0, words - 1024, size=6):
            ws.append((int(r), int(r) + 1024))
        win[k] = ws
    return win


def test_lulesh250_full_size_sampled_parity():
    import torch
    from oracle import Oracle
    from paper_conf_ipps_pirkelbauerlvl20_b200 import apps, xpl
    from xplgen import lulesh as L

    spec = L.lulesh_spec(S)
    ar = apps.Arena(spec)
    topo = L.topology(S, 0x58504C05)
    apps.lulesh_prepare(ar, S, topo)
    win = _windows(S, np.random.default_rng(0x58504C05))
    words = [(sp[1] + 3) // 4 for sp in spec]
    st = torch.cuda.Stream()
    hc = torch.zeros(1, dtype=torch.int64, device="cuda")
    pool = sum(words) + STEPS * 54 * S ** 3 + (1 << 24)
    assert pool > (1 << 31)  # word indices beyond 2^31
    dumps, full_counts = {}, {}
    with xpl.Context(pool_words=pool, max_rows=64) as ctx:
        run = apps.Run(ctx, st.cuda_stream, params=PARAMS, out_cap=64 * (STEPS + 1), diag_reset=False,
                       keep_allocs=True)
        tmps = apps.lulesh(run, ar, S, STEPS, hc)
        got = run.reports()
        for k, ws in win.items():
            dumps[k] = [ctx.shadow_dump(ar.addrs[2 + k], w0, w1 - w0) for w0, w1 in ws]
        dumps["dom"] = ctx.shadow_dump(ar.addrs[0], 0, words[0])
        for i in range(len(spec)):
            c = np.zeros(9, np.int64)
            for w0 in range(0, words[i], 1 << 27):
                r = ctx.shadow_dump(ar.addrs[i], w0, min(1 << 27, words[i] - w0))
                cpu, gpu = (r & 0x34) != 0, (r & 0xC8) != 0
                c += [np.count_nonzero(r & b) for b in (0x04, 0x08, 0x10, 0x40, 0x20, 0x80)] + \
                     [np.count_nonzero(cpu | gpu), np.count_nonzero(gpu),
                      np.count_nonzero(cpu & gpu & ((r & 0x0C) != 0))]
            full_counts[i] = c
    assert len(got) == STEPS
    last = got[-1]
    for i in range(len(spec)):  # property at full size: counters = popcounts of the shadow (D21)
        row = last[i]
        assert row["words"] == words[i]
        assert [row[f] for f in ("w_c", "w_g", "r_cc", "r_cg", "r_gc", "r_gg", "any_acc", "gpu_acc",
                                 "alternating")] == full_counts[i].tolist(), spec[i][0]
    ops, hooks = L.lulesh_trace(ar.addrs, spec, S, STEPS, topo, PARAMS, tmps, windows=win, reset=0, final=False)
    assert hooks is None
    # (a) the two complete rows: a replay restricted to dom and dt_block (ids 0, 1:
    # registered first), so the oracle's diagnose does not walk 3e9 other words
    lo, hi = ar.addrs[0], ar.addrs[1] + spec[1][1]
    small = []
    for op in ops:
        if op[0] in ("HB", "DB"):
            a = np.asarray(op[1], np.uint64)
            m = (a >= lo) & (a < hi) & ((a < ar.addrs[0] + spec[0][1]) | (a >= ar.addrs[1]))
            small.append((op[0], a[m], np.asarray(op[2])[m], np.asarray(op[3])[m]))
        elif op[0] in ("H", "D"):
            if ar.addrs[0] <= op[1] < ar.addrs[0] + spec[0][1] or ar.addrs[1] <= op[1] < hi:
                small.append(op)
        elif op[0] in ("REG", "FREE"):
            if op[1] in (ar.addrs[0], ar.addrs[1]):
                small.append(op)
        else:
            small.append(op)
    o2 = Oracle()
    exp = [r for r in map(o2.op, small) if r is not None]
    assert len(exp) == len(got)
    # (b) the sampled words: the whole sampled trace without its diagnoses (with
    # reset = 0 a diagnose changes no record, D25)
    o = Oracle()
    for op in ops:
        if op[0] != "DIAG":
            o.op(op)
    for d, (g, e) in enumerate(zip(got, exp)):
        for i in (0, 1):  # dom, dt_block: complete rows
            diff = {f: (g[i][f], e[i][f]) for f in e[i] if g[i][f] != e[i][f]}
            assert not diff, (d, spec[i][0], diff)
    assert np.array_equal(dumps["dom"] & 0xFD, np.array([o.peek(0, w) for w in range(words[0])], np.uint8))
    for k, ws in win.items():
        for (w0, w1), gd in zip(ws, dumps[k]):
            ed = np.array([o.peek(2 + k, w) for w in range(w0, w1)], np.uint8)
            bad = np.nonzero((gd & 0xFD) != ed)[0]
            assert bad.size == 0, (L.NAMES[k], w0 + int(bad[0]), int(gd[bad[0]]), int(ed[bad[0]]))

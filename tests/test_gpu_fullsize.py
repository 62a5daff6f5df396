"""Parity at BASELINE.json's full sizes, in the launch configuration bench.py
times (configs[1]: hotspot 1024^2 x 20, backprop 640K x 16, bfs 1M x 6,
nw 2048^2; resident data, a diagnose after every iteration and at the end).

Every report row of every diagnose is compared with the oracle.  The oracle is
run per allocation group in parallel processes: a word's record depends only on
the events that touch that word, so replaying the trace filtered to a group of
allocations gives exactly the rows of that group (SURVEY §8(d) "partitioned by
allocation").  Slow (minutes of host CPU); part of -m gpu.
"""
import multiprocessing as mp
import os

import numpy as np
import pytest

pytestmark = [pytest.mark.gpu, pytest.mark.slow]

_TRACE = None  # shared with forked workers


def _filter(ops, keep_ranges):
    lo = np.array([a for a, _ in keep_ranges], dtype=np.uint64)
    hi = np.array([a + n for a, n in keep_ranges], dtype=np.uint64)
    order = np.argsort(lo)
    lo, hi = lo[order], hi[order]

    def inside(addr):
        addr = np.asarray(addr, dtype=np.uint64)
        k = np.searchsorted(lo, addr, side="right") - 1
        ok = k >= 0
        kk = np.clip(k, 0, len(lo) - 1)
        return ok & (addr < hi[kk])

    out = []
    for op in ops:
        t = op[0]
        if t in ("HB", "DB"):
            m = inside(op[1])
            if m.any():
                out.append((t, op[1][m], op[2][m], op[3][m]))
        elif t in ("H", "D"):
            if inside([op[1]])[0]:
                out.append(op)
        elif t == "X":
            if inside([op[2]])[0] or inside([op[3]])[0]:
                out.append(op)
        else:
            out.append(op)
    return out


def _work(args):
    ids, ranges = args
    from oracle import run_trace
    res = run_trace(_filter(_TRACE, ranges))
    return [[r for r in d if r["id"] in ids] for d in res]


def partitioned_oracle(ops, groups):
    """groups: list of lists of (allocation id, base, bytes)."""
    global _TRACE
    _TRACE = ops
    jobs = [({i for i, _, _ in g}, [(b, n) for _, b, n in g]) for g in groups]
    with mp.get_context("fork").Pool(min(len(jobs), os.cpu_count() or 4)) as pool:
        parts = pool.map(_work, jobs)
    _TRACE = None
    merged = []
    for k in range(len(parts[0])):
        rows = sorted((r for p in parts for r in p[k]), key=lambda r: r["id"])
        merged.append(rows)
    return merged


def compare(got, exp):
    assert len(got) == len(exp), (len(got), len(exp))
    for k, (g, e) in enumerate(zip(got, exp)):
        assert [r["id"] for r in g] == [r["id"] for r in e], f"diag {k}: row ids differ"
        for gr, er in zip(g, e):
            diff = {f: (gr[f], er[f]) for f in er if gr[f] != er[f]}
            assert not diff, f"diag {k} row {er['id']}: (gpu, oracle) {diff}"


def one_per_allocation(spec, addrs):
    return [[(i, a, s[1])] for i, (a, s) in enumerate(zip(addrs, spec))]


@pytest.fixture(scope="module")
def env():
    import torch
    assert torch.cuda.is_available()
    import bench
    from paper_conf_ipps_pirkelbauerlvl20_b200 import apps, xpl
    return torch, apps, xpl, bench


def run_app(env, spec, fn, *args, do_copies=False, pool=1 << 27):
    torch, apps, xpl, bench = env
    s = torch.cuda.Stream()
    with xpl.Context(pool_words=pool, max_rows=64) as ctx:
        run = apps.Run(ctx, s.cuda_stream, do_copies=do_copies, diag_each=True, params=bench.PARAMS)
        r = fn(run, *args)
        return run.reports(), r


def test_hotspot_full(env):
    torch, apps, xpl, bench = env
    from xplgen import rodinia
    rows, cols, iters = bench.HOT
    spec = rodinia.hotspot_spec(rows, cols)
    ar = apps.Arena(spec)
    rodinia.fill_inputs("hotspot", ar.host_views(), 0x58504C01)
    got, _ = run_app(env, spec, apps.hotspot, ar, rows, cols, iters)
    ops = rodinia.hotspot_trace(ar.addrs, spec, rows, cols, iters, True, bench.PARAMS)
    compare(got, partitioned_oracle(ops, one_per_allocation(spec, ar.addrs)))


def test_backprop_full(env):
    torch, apps, xpl, bench = env
    from xplgen import rodinia
    spec = rodinia.backprop_spec(*bench.BACKPROP)
    ar = apps.Arena(spec)
    got, _ = run_app(env, spec, apps.backprop, ar, *bench.BACKPROP)
    ops = rodinia.backprop_trace(ar.addrs, spec, *bench.BACKPROP, bench.PARAMS)
    compare(got, partitioned_oracle(ops, one_per_allocation(spec, ar.addrs)))


def test_bfs_full(env):
    torch, apps, xpl, bench = env
    from xplgen import rodinia
    n, deg = bench.BFS
    spec = rodinia.bfs_spec(n, deg)
    ar = apps.Arena(spec)
    edges = rodinia.bfs_graph(n, deg, 0x58504C02)
    apps.bfs_prepare(ar, n, deg, edges, resident=True)
    hc = torch.zeros(1, dtype=torch.int64, device="cuda")
    got, levels = run_app(env, spec, apps.bfs, ar, n, deg, hc)
    ops, lv, hooks = rodinia.bfs_trace(ar.addrs, spec, n, deg, edges, True, bench.PARAMS)
    assert levels == lv and int(hc.item()) == hooks
    compare(got, partitioned_oracle(ops, one_per_allocation(spec, ar.addrs)))


def test_nw_full(env):
    torch, apps, xpl, bench = env
    from xplgen import rodinia
    n, pen = bench.NW
    spec = rodinia.nw_spec(n)
    ar = apps.Arena(spec)
    inp = rodinia.nw_inputs(n, pen, 0x58504C03)
    rodinia.nw_fill_host(ar.host_views(), spec, inp, n)
    got, _ = run_app(env, spec, apps.nw, ar, n, pen, inp["blosum"])
    ops = rodinia.nw_trace(ar.addrs, spec, n, pen, inp, bench.PARAMS)
    compare(got, partitioned_oracle(ops, one_per_allocation(spec, ar.addrs)))

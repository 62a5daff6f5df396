"""Brute-force pin: the oracle's record state machine against the independent
history evaluator (tests/history_ref.py) on every trace of one 2-word
allocation with up to 3 host/GPU segments of up to 2 ops from {R,W,RW}x{w0,w1},
with and without reset-diagnoses between segments (SURVEY.md §8(c) "pins"),
plus seeded random traces with transfers, frees, unaligned and multi-word
accesses, deferred host events and random diagnose parameters.
"""
import itertools

import numpy as np
import pytest

from oracle import run_trace
from tests.history_ref import evaluate
from xplgen.trace import DEVICE, HOST, MANAGED, SEG_OPS, enumerated_trace, random_trace, schedules

FIELDS = None


def compare(ops):
    got = run_trace(ops)
    exp = evaluate(ops)
    assert len(got) == len(exp)
    for k, (g, e) in enumerate(zip(got, exp)):
        assert len(g) == len(e), f"diag {k}: {len(g)} rows vs {len(e)}"
        for gr, er in zip(g, e):
            diff = {f: (gr[f], er[f]) for f in er if gr[f] != er[f]}
            assert not diff, f"diag {k} row {er['id']}: (oracle, history) {diff}"


@pytest.mark.parametrize("schedule", schedules(2), ids=lambda s: "".join(s[0]) + "".join("d" if x else "-" for x in s[1]))
def test_exhaustive_two_segments(schedule):
    nseg = len(schedule[0])
    asg = list(itertools.product(SEG_OPS, repeat=nseg))
    for kind in (MANAGED, DEVICE):
        compare(enumerated_trace(schedule, asg, kind=kind))


@pytest.mark.parametrize("schedule", [s for s in schedules(3) if len(s[0]) == 3],
                         ids=lambda s: "".join(s[0]) + "".join("d" if x else "-" for x in s[1]))
def test_sampled_three_segments(schedule):
    rng = np.random.default_rng(0x58504C00)
    allasg = list(itertools.product(range(len(SEG_OPS)), repeat=3))
    pick = rng.choice(len(allasg), size=2500, replace=False)
    asg = [tuple(SEG_OPS[i] for i in allasg[p]) for p in pick]
    compare(enumerated_trace(schedule, asg))


@pytest.mark.parametrize("seed", range(40))
def test_random_traces(seed):
    compare(random_trace(0x58504C00 + seed, n_allocs=5, n_steps=50, max_words=64))


def test_lulesh_sampled_twin_equals_full_twin():
    """The sampled LULESH twin (cfg5 full-size parity: only the events of chosen
    word windows, repeats inside an epoch dropped, temporaries left out) leaves
    every sampled word -- and every word of dom and dt_block, whose rows it
    reproduces exactly -- with the record the full trace gives."""
    from oracle import Oracle
    from xplgen import lulesh as L
    from xplgen.rodinia import layout
    s = 5
    spec = L.lulesh_spec(s)
    addrs, _, _ = layout(spec, 1 << 40, 1 << 44, 1 << 36)
    topo = L.topology(s, 0x58504C05)
    tmps = [((1 << 50) + (2 * i << 30), (1 << 50) + ((2 * i + 1) << 30)) for i in range(3)]
    win = {k: [(0, 7), (31, 45), (L.slot_bytes(s, k) // 4 - 5, L.slot_bytes(s, k) // 4)] for k in range(0, 48, 2)}
    full, _ = L.lulesh_trace(addrs, spec, s, 3, topo, (50, 0, 256), tmps, reset=0, final=False)
    samp, hooks = L.lulesh_trace(addrs, spec, s, 3, topo, (50, 0, 256), tmps, windows=win, reset=0, final=False)
    assert hooks is None
    assert sum(len(op[1]) for op in samp if op[0] in ("DB", "HB")) < \
        sum(len(op[1]) for op in full if op[0] in ("DB", "HB")) // 5
    o1, o2 = Oracle(), Oracle()
    d1 = [r for r in map(o1.op, full) if r is not None]
    d2 = [r for r in map(o2.op, samp) if r is not None]
    for a, b in zip(d1, d2):
        assert a[0] == b[0] and a[1] == b[1]  # dom, dt_block: complete rows
    for k, ws in win.items():
        for w0, w1 in ws:
            for w in range(w0, w1):
                assert o1.peek(2 + k, w) == o2.peek(2 + k, w), (k, w)
    for w in range(L.DOM_BYTES // 4):
        assert o1.peek(0, w) == o2.peek(0, w)


def test_page_view_invariants():
    """NEXT-3 page view tied to the (pinned) diagnose counters: with one word per
    page the page counts are the per-word classes (gpu_pages = gpu_acc, CPU or
    GPU pages = any_acc, alternating_pages = alternating); with one page per
    allocation they are indicators of the same counters; false-shared pages
    never exceed shared ones; flags only on managed allocations."""
    from oracle import run_trace
    from xplgen.trace import random_trace, with_pages
    for seed in range(12):
        ops = with_pages(random_trace(0x58504C40 + seed, n_allocs=5, n_steps=70, max_words=600),
                          (1, 7, 1 << 40), seed)
        res = run_trace(ops)
        k = 0
        while k < len(res):
            p1, p7, pbig, diag = res[k:k + 4]
            k += 4
            live = {r["id"]: r for r in diag if r["live"]}
            assert [r["id"] for r in p1] == sorted(live)
            for a, b, c in zip(p1, p7, pbig):
                d = live[a["id"]]
                assert a["pages"] == d["words"] and c["pages"] == 1 and b["pages"] == -(-d["words"] // 7)
                assert a["gpu_pages"] == d["gpu_acc"]
                assert a["cpu_pages"] + a["gpu_pages"] - a["shared_pages"] == d["any_acc"]
                assert a["alternating_pages"] == d["alternating"] and a["false_shared_pages"] == 0
                assert c["gpu_pages"] == int(d["gpu_acc"] > 0) and c["alternating_pages"] == int(d["alternating"] > 0)
                assert c["cpu_pages"] + c["gpu_pages"] - c["shared_pages"] == int(d["any_acc"] > 0)
                for x in (a, b, c):
                    assert x["false_shared_pages"] <= x["shared_pages"] <= min(x["cpu_pages"], x["gpu_pages"])
                    assert x["alternating_pages"] <= x["shared_pages"] - x["false_shared_pages"]
                    if d["kind"] != 1:
                        assert x["flags"] == 0
                    assert bool(x["flags"] & 1) == (d["kind"] == 1 and x["false_shared_pages"] > 0)

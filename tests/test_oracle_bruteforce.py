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

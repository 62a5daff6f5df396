"""The record-preserving reductions tools/golden_fullsize.py applies before the
oracle computes the stored full-size expectations (tests/golden/fullsize/):
on small instances of the same programs the reduced trace must give exactly
the reports of the plain trace (every field), and the LULESH-shaped program's
reports must be periodic after timestep 2 (the premise of checking timesteps
4..100 against timestep 3)."""
import os
import sys

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, os.path.join(ROOT, "tools"))

import golden_fullsize as G  # noqa: E402
from oracle import run_trace  # noqa: E402


def _strip(diags):
    return [[{f: v for f, v in r.items() if f != "base"} for r in d] for d in diags]


@pytest.mark.parametrize("n,m", [(40, 70), (129, 64)])
def test_sw_reduced_equals_plain(n, m):
    from xplgen import sw
    from xplgen.rodinia import layout
    spec = sw.sw_spec(n, m)
    addrs, _, _ = layout(spec, 0, 0, 1 << 40)
    inp = sw.sw_inputs(n, m, 7)
    ops = sw.sw_trace(addrs, spec, n, m, 1, 16, 32, inp, G.PARAMS[:2] + (4,))
    assert _strip(run_trace(ops)) == G.replay(G.reduced(ops))


def test_lulesh_reduced_equals_plain_and_periodic():
    ops, meta = G.cfg4_ops(s=5, steps=6)
    ops = list(ops)
    plain = _strip(run_trace(ops))
    red = G.replay(G.reduced(ops))
    assert plain == red
    assert len(red) == 7  # 6 timesteps + the final diagnose after the frees

    def persistent(d):  # temporaries (ids >= 50) are new rows every timestep
        return [r for r in d if r["id"] < 50]

    def temps(d):
        return [{f: v for f, v in r.items() if f != "id"} for r in d if r["id"] >= 50]
    for t in range(3, 6):  # reports of timesteps 4..6 equal timestep 3's (periodic after timestep 2)
        assert persistent(red[t]) == persistent(red[2])
        assert temps(red[t]) == temps(red[2])
    assert persistent(red[1]) == persistent(red[2])  # (already periodic from timestep 2 on)
    # the final diagnose: every allocation freed after a reset -> no access in the interval
    assert all(r["any_acc"] == 0 and r["live"] == 0 for r in red[6])


def test_cfg5_partition_merge_equals_plain():
    """cfg5's expectations are replayed partitioned by allocation (the force
    temporary in word windows) and merged; on a small mesh the merged reports
    must equal the plain replay of the whole program, every field."""
    from xplgen import lulesh as L
    from xplgen.rodinia import layout
    s, steps = 6, 3
    fw = 24 * s ** 3 * 2
    cut = [0, (fw // 3 + 5) & ~1, (2 * fw // 3 + 1) & ~1, fw]  # (windows cut between 8-byte elements)
    jobs = [(f"g{i}", g, None) for i, g in enumerate(G.CFG5_GROUPS)]
    jobs += [(f"force{i}", (), {0: [(cut[i], cut[i + 1])]}) for i in range(3)]
    jobs.append(("dvdx", (), {1: [(0, 3 * s ** 3 * 2)]}))
    parts = []
    for name, slots, tmp in jobs:
        keep = {0, 1} | {2 + k for k in slots}
        d = G.replay(G.reduced(G.cfg5_ops(slots, tmp, s=s, steps=steps)))
        parts.append({"name": name, "tmp": tmp,
                      "diagnoses": [[r for r in x if r["id"] in keep or (tmp and r["id"] >= 50)] for x in d]})
    got = G.cfg5_merge(parts)
    spec = L.lulesh_spec(s)
    addrs, _, _ = layout(spec, 0, 0, 1 << 40)
    tmps = [((1 << 44) + t * (1 << 36), (1 << 44) + t * (1 << 36) + (1 << 35)) for t in range(steps)]
    plain = _strip(run_trace(list(L.lulesh_trace_iter(addrs, spec, s, steps, L.topology(s, 0x58504C05),
                                                      G.PARAMS, tmps))))
    assert got == plain

"""Full-size parity of BASELINE.json configs[2] (cfg3, Smith-Waterman 16K x 16K)
and configs[3] (cfg4, LULESH-shaped 100^3 x 100 timesteps), in the launch
configuration bench.py times, against expectations the ORACLE computed
(tests/golden/fullsize/*.json, written by tools/golden_fullsize.py, which calls
only oracle/ and the seeded CPU twins; the full traces take the oracle tens of
minutes, too long for a test).  Every field of every report row is compared
except `base` (the golden run used synthetic addresses).

cfg3: all 32 diagnoses of the 32,767-epoch program (a diagnose every 1,024
      anti-diagonals, the final one after the traceback and frees).
cfg4: the golden holds the first 3 timesteps + the final diagnose (SURVEY §8(d):
      the program is periodic after timestep 2 -- tests/test_golden_fullsize_cpu.py
      pins that on the oracle); timesteps 1-3 are compared with it, timesteps
      4..100 with timestep 3 (temporaries: new ids every timestep), the final
      diagnose with the golden final one; and the complete rows of `dom` (the
      Fig. 4 object) and `dt_block` of all 100 diagnoses against the oracle's
      replay of the sampled twin (every event of those two allocations).
cfg5: LULESH-shaped 250^3 x 100 timesteps on one GPU against the oracle's
      replay partitioned by allocation (timesteps 1-2 + the final diagnose;
      periodic from timestep 2 on)."""
import json
import os

import numpy as np
import pytest

pytestmark = [pytest.mark.gpu, pytest.mark.slow]

GOLD = os.path.join(os.path.dirname(os.path.abspath(__file__)), "golden", "fullsize")


def _load(name):
    p = os.path.join(GOLD, name + ".json")
    if not os.path.exists(p):
        pytest.skip(f"{p} not generated yet (tools/golden_fullsize.py {name})")
    with open(p) as f:
        return json.load(f)


def _strip(d):
    return [{f: v for f, v in r.items() if f != "base"} for r in d]


def _diff(g, e):
    return {f: (g[f], e[f]) for f in e if g[f] != e[f]}


def test_cfg4_lulesh100_full_size():
    import torch
    from oracle import run_trace
    from paper_conf_ipps_pirkelbauerlvl20_b200 import apps, xpl
    from xplgen import lulesh as L
    gold = _load("cfg4")
    s, T = 100, 100
    params = tuple(gold["meta"]["params"])
    spec = L.lulesh_spec(s)
    ar = apps.Arena(spec)
    topo = L.topology(s, gold["meta"]["seed"])
    apps.lulesh_prepare(ar, s, topo)
    hc = torch.zeros(1, dtype=torch.int64, device="cuda")
    st = torch.cuda.Stream()
    with xpl.Context(pool_words=1 << 28, max_rows=64) as ctx:  # bench.py's context
        run = apps.Run(ctx, st.cuda_stream, params=params, out_cap=64 * (T + 2))
        tmps = apps.lulesh(run, ar, s, T, hc)
        got = [_strip(d) for d in run.reports()]
    exp = gold["diagnoses"]
    assert len(exp) == 4 and len(got) == T + 1
    for t in range(3):  # timesteps 1-3: every row
        assert len(got[t]) == len(exp[t])
        for g, e in zip(got[t], exp[t]):
            assert not _diff(g, e), (t, e["id"], _diff(g, e))
    per = lambda d: [r for r in d if r["id"] < 50]
    tmp = lambda d: [{f: v for f, v in r.items() if f != "id"} for r in d if r["id"] >= 50]
    for t in range(3, T):  # periodic: timestep t+1 = timestep 3
        assert per(got[t]) == per(exp[2]), t
        assert tmp(got[t]) == tmp(exp[2]), t
        assert [r["id"] for r in got[t] if r["id"] >= 50] == [50 + 2 * t, 51 + 2 * t]
    for g, e in zip(got[T], exp[3]):  # the final diagnose after the frees
        assert not _diff(g, e), ("final", e["id"], _diff(g, e))
    # dom and dt_block, complete, in all 100 diagnoses (sampled twin: only their events)
    ops, _ = L.lulesh_trace(ar.addrs, spec, s, T, topo, params, tmps, windows={}, reset=1, final=True)
    small = []
    lo0, hi0 = ar.addrs[0], ar.addrs[0] + spec[0][1]
    lo1, hi1 = ar.addrs[1], ar.addrs[1] + spec[1][1]
    for op in ops:
        if op[0] in ("HB", "DB"):
            a = np.asarray(op[1], np.uint64)
            m = ((a >= lo0) & (a < hi0)) | ((a >= lo1) & (a < hi1))
            small.append((op[0], a[m], np.asarray(op[2])[m], np.asarray(op[3])[m]))
        elif op[0] in ("REG", "FREE"):
            if op[1] in (lo0, lo1):
                small.append(op)
        elif op[0] in ("H", "D"):
            if lo0 <= op[1] < hi0 or lo1 <= op[1] < hi1:
                small.append(op)
        else:
            small.append(op)
    ex2 = run_trace(small)
    assert len(ex2) == T + 1
    for t in range(T + 1):
        for i in (0, 1):
            e = {f: v for f, v in ex2[t][i].items() if f != "base"}
            assert not _diff(got[t][i], e), (t, i, _diff(got[t][i], e))
    # Fig. 4: dom after every timestep after the first
    for t in range(1, T):
        d = got[t][0]
        assert (d["w_c"], d["w_g"], d["r_cc"], d["density_pct_gpu"], d["alternating"]) == (27, 0, 680, 9, 18)


def test_cfg3_sw16k_full_size():
    import torch
    from paper_conf_ipps_pirkelbauerlvl20_b200 import apps, xpl
    from xplgen import sw
    gold = _load("cfg3")
    m = gold["meta"]
    n, mm = m["n"], m["m"]
    spec = sw.sw_spec(n, mm)
    ar = apps.Arena(spec)
    inp = sw.sw_inputs(n, mm, m["seed"])
    st = torch.cuda.Stream()
    with xpl.Context(pool_words=1 << 29, max_rows=16) as ctx:  # bench.py's context
        run = apps.Run(ctx, st.cuda_stream, params=tuple(m["params"]))
        apps.sw(run, ar, n, mm, m["per_diagonal"], m["tb_every"], m["diag_every"], inp)
        got = [_strip(d) for d in run.reports()]
        assert run.r.epochs >= n + mm - 1
    exp = gold["diagnoses"]
    assert len(got) == len(exp)
    for t, (gd, ed) in enumerate(zip(got, exp)):
        assert len(gd) == len(ed)
        for g, e in zip(gd, ed):
            assert not _diff(g, e), (t, e["id"], _diff(g, e))
    assert all(d[2]["words"] == (n + 1) * (mm + 1) for d in got)


def test_cfg5_lulesh250_full_size():
    """configs[4] (cfg5) at full size on one B200 -- LULESH-shaped 250^3 x 100
    timesteps, 2.3e9 shadow words per timestep -- against the oracle's
    partitioned replay (tests/golden/fullsize/cfg5.json, tools/golden_fullsize.py
    cfg5): timesteps 1-2 every row, 3..100 equal to timestep 2 (periodic), the
    final diagnose every row."""
    import torch
    from paper_conf_ipps_pirkelbauerlvl20_b200 import apps, xpl
    from xplgen import lulesh as L
    gold = _load("cfg5")
    s, T = 250, 100
    params = tuple(gold["meta"]["params"])
    steps = gold["meta"]["steps"]
    spec = L.lulesh_spec(s)
    ar = apps.Arena(spec)
    apps.lulesh_prepare(ar, s, L.topology(s, gold["meta"]["seed"]))
    hc = torch.zeros(1, dtype=torch.int64, device="cuda")
    st = torch.cuda.Stream()
    with xpl.Context(pool_words=2_500_000_000, max_rows=64) as ctx:  # bench.py's cfg5 context
        run = apps.Run(ctx, st.cuda_stream, params=params, out_cap=64 * (T + 2))
        apps.lulesh(run, ar, s, T, hc)
        got = [_strip(d) for d in run.reports()]
    exp = gold["diagnoses"]
    assert len(exp) == steps + 1 and len(got) == T + 1
    for t in range(steps):
        assert [r["id"] for r in got[t]] == [r["id"] for r in exp[t]]
        for g, e in zip(got[t], exp[t]):
            assert not _diff(g, e), (t, e["id"], _diff(g, e))
    per = lambda d: [r for r in d if r["id"] < 50]
    tmp = lambda d: [{f: v for f, v in r.items() if f != "id"} for r in d if r["id"] >= 50]
    for t in range(steps, T):
        assert per(got[t]) == per(exp[steps - 1]), t
        assert tmp(got[t]) == tmp(exp[steps - 1]), t
    for g, e in zip(got[T], exp[steps]):
        assert not _diff(g, e), ("final", e["id"], _diff(g, e))

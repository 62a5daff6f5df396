"""GPU parity of the instrumented Rodinia-shaped programs (configs[1]): the native
app (csrc/work_rodinia.cu) runs through the C-ABI; its CPU twin (xplgen/rodinia.py)
is replayed by the oracle at the SAME addresses; every report of every diagnose
must match bit-exactly.  Sizes span several diagnose tiles with ragged tails."""
import numpy as np
import pytest

from oracle import run_trace as oracle_run

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def env():
    import torch
    assert torch.cuda.is_available()
    from paper_conf_ipps_pirkelbauerlvl20_b200 import apps, xpl
    return torch, apps, xpl


def compare(got, exp):
    assert len(got) == len(exp), (len(got), len(exp))
    for k, (g, e) in enumerate(zip(got, exp)):
        assert len(g) == len(e), f"diag {k}: {len(g)} rows vs {len(e)}"
        for gr, er in zip(g, e):
            diff = {f: (gr[f], er[f]) for f in er if gr[f] != er[f]}
            assert not diff, f"diag {k} row {er['id']}: (gpu, oracle) {diff}"


@pytest.mark.parametrize("rows,cols,iters", [(8, 40, 3), (67, 130, 4), (256, 300, 3)])
@pytest.mark.parametrize("params", [(50, 0, 256), (30, 1000, 8)])
def test_hotspot(env, rows, cols, iters, params):
    torch, apps, xpl = env
    from xplgen import rodinia
    spec = rodinia.hotspot_spec(rows, cols)
    ar = apps.Arena(spec)
    rodinia.fill_inputs("hotspot", ar.host_views(), 0x58504C01)
    s = torch.cuda.Stream()
    with xpl.Context(pool_words=1 << 24) as ctx:
        run = apps.Run(ctx, s.cuda_stream, do_copies=True, diag_each=True, params=params)
        apps.hotspot(run, ar, rows, cols, iters)
        got = run.reports()
        assert run.r.dev_accesses == iters * rodinia.hotspot_accesses(rows, cols)
    exp = oracle_run(rodinia.hotspot_trace(ar.addrs, spec, rows, cols, iters, True, params))
    compare(got, exp)


@pytest.mark.parametrize("n_in", [64, 1024, 40960])
def test_backprop(env, n_in):
    torch, apps, xpl = env
    from xplgen import rodinia
    spec = rodinia.backprop_spec(n_in, 16)
    ar = apps.Arena(spec)
    rodinia.fill_inputs("backprop", ar.host_views(), 0x58504C01)
    s = torch.cuda.Stream()
    params = (50, 0, 256)
    with xpl.Context(pool_words=1 << 25) as ctx:
        run = apps.Run(ctx, s.cuda_stream, do_copies=bool(n_in % 2048), params=params)
        apps.backprop(run, ar, n_in, 16)
        got = run.reports()
    exp = oracle_run(rodinia.backprop_trace(ar.addrs, spec, n_in, 16, params))
    compare(got, exp)
    # Table II: output_hidden_cuda unused; input_cuda copied back unmodified
    rows = {r["id"]: r for r in got[-1]}
    assert rows[6]["flags"] & 16
    if n_in + 1 >= params[2]:
        assert rows[5]["flags"] & 8


@pytest.mark.parametrize("n,resident", [(1000, False), (5000, True), (70000, False)])
def test_bfs(env, n, resident):
    torch, apps, xpl = env
    from xplgen import rodinia
    deg = 6
    spec = rodinia.bfs_spec(n, deg)
    ar = apps.Arena(spec)
    edges = rodinia.bfs_graph(n, deg, 0x58504C02 + n)
    apps.bfs_prepare(ar, n, deg, edges, resident)
    s = torch.cuda.Stream()
    params = (50, 0, 64)
    hc = torch.zeros(1, dtype=torch.int64, device="cuda")
    with xpl.Context(pool_words=1 << 24) as ctx:
        run = apps.Run(ctx, s.cuda_stream, do_copies=not resident, diag_each=True, params=params)
        levels = apps.bfs(run, ar, n, deg, hc)
        got = run.reports()
    ops, lv, hooks = rodinia.bfs_trace(ar.addrs, spec, n, deg, edges, True, params)
    assert levels == lv
    assert int(hc.item()) == hooks
    compare(got, oracle_run(ops))


@pytest.mark.parametrize("n,resident", [(64, False), (256, True), (512, False)])
def test_nw(env, n, resident):
    torch, apps, xpl = env
    from xplgen import rodinia
    spec = rodinia.nw_spec(n)
    ar = apps.Arena(spec)
    inp = rodinia.nw_inputs(n, 10, 0x58504C03 + n)
    rodinia.nw_fill_host(ar.host_views(), spec, inp, n)
    s = torch.cuda.Stream()
    params = (50, 1024, 16)
    with xpl.Context(pool_words=1 << 24) as ctx:
        run = apps.Run(ctx, s.cuda_stream, do_copies=not resident, params=params)
        apps.nw(run, ar, n, 10, inp["blosum"])
        got = run.reports()
        assert run.r.dev_accesses == rodinia.nw_accesses(n)
    compare(got, oracle_run(rodinia.nw_trace(ar.addrs, spec, n, 10, inp, params)))
    if not resident:  # the kernels computed the DP the twin expects
        out = ar.view("output_itemsets").view(np.int32).reshape(n + 1, n + 1)
        assert np.array_equal(out[1:, 1:], inp["dp"][1:, 1:])


@pytest.mark.parametrize("n,m,per_diag,tb_every,diag_every", [
    (128, 128, 0, 0, 0),          # cfg1 SW-128: one launch, 4 epochs
    (128, 128, 2, 0, 0),          # cfg1 with a device-side epoch split per anti-diagonal (NEXT-2)
    (37, 90, 2, 0, 0),
    (40, 70, 1, 16, 32),       # cfg3 shape: per-diagonal launches, traceback + diagnose points
    (300, 257, 1, 64, 128)])
def test_smith_waterman(env, n, m, per_diag, tb_every, diag_every):
    torch, apps, xpl = env
    from xplgen import sw
    spec = sw.sw_spec(n, m)
    ar = apps.Arena(spec)
    inp = sw.sw_inputs(n, m, 0x58504C04 + n)
    s = torch.cuda.Stream()
    params = (50, 0, 8)
    with xpl.Context(pool_words=1 << 22) as ctx:
        run = apps.Run(ctx, s.cuda_stream, params=params)
        tb = apps.sw(run, ar, n, m, per_diag, tb_every, diag_every, inp)
        got = run.reports()
        assert run.r.dev_accesses == sw.sw_accesses(n, m, per_diag)
    H = sw.sw_dp(inp["a"], inp["b"])
    assert tb == sw.sw_traceback(H, inp["a"], inp["b"])[3]
    if per_diag == 1:  # (the single-launch programs re-zero H at the end)
        assert np.array_equal(ar.view("H").view(np.int32).reshape(n + 1, m + 1), H)
    compare(got, oracle_run(sw.sw_trace(ar.addrs, spec, n, m, per_diag, tb_every, diag_every, inp, params)))
    if per_diag == 2:
        # split epochs: the wavefront reads its own earlier diagonals as G>G; only
        # the CPU's boundary zeros (row 0 and column 0) are C>G (Fig. 7)
        h = got[-1][2]
        assert h["w_g"] == n * m and h["r_cg"] == n + m + 1 and h["r_gg"] > 0
    if not per_diag:
        # cfg1 under the snapshot reading (D5): one launch sees only the pre-epoch
        # (CPU) values, so no read of H is G>G although the wavefront reads its own output
        h = got[-1][2]
        assert h["w_g"] == n * m and h["r_gg"] == 0 and h["r_cg"] == (n + 1) * (m + 1) - 1


def test_lulesh_layout_matches_twin(env):
    torch, apps, xpl = env
    from xplgen import lulesh as L
    assert apps.lulesh_layout() == [L.DOM_BYTES, L.OFF_NUMELEM, L.OFF_DT, L.OFF_TIME, L.OFF_CYCLE,
                                    L.OFF_DTC, L.OFF_DTH, L.OFF_MISC, L.OFF_PARAMS]


@pytest.mark.parametrize("s,steps", [(8, 3), (5, 2), (13, 2)])
def test_lulesh(env, s, steps):
    torch, apps, xpl = env
    from xplgen import lulesh as L
    spec = L.lulesh_spec(s)
    ar = apps.Arena(spec)
    topo = L.topology(s, 0x58504C05)
    apps.lulesh_prepare(ar, s, topo)
    st = torch.cuda.Stream()
    params = (50, 0, 256)
    hc = torch.zeros(1, dtype=torch.int64, device="cuda")
    with xpl.Context(pool_words=1 << 24) as ctx:
        run = apps.Run(ctx, st.cuda_stream, params=params)
        tmps = apps.lulesh(run, ar, s, steps, hc)
        got = run.reports()
    ops, hooks = L.lulesh_trace(ar.addrs, spec, s, steps, topo, params, tmps)
    assert int(hc.item()) == hooks
    exp = oracle_run(ops)
    compare(got, exp)
    if s == 8:
        # Fig. 4, "after the second iteration": dom C=27, G=0, C>C=680,
        # density 9 %, 18 alternating; (dom)->m_p C=0, G=1024, C>C=0, G>G=1024, 100 %, 0
        dom = got[1][0]
        assert (dom["w_c"], dom["w_g"], dom["r_cc"], dom["density_pct_gpu"], dom["alternating"]) == (27, 0, 680, 9, 18)
        mp = got[1][2 + L.P]
        assert (mp["words"], mp["w_c"], mp["w_g"], mp["r_cc"], mp["r_gg"], mp["density_pct_gpu"],
                mp["alternating"]) == (1024, 0, 1024, 0, 1024, 100, 0)


def test_twin_runs_without_xpl(env):
    torch, apps, xpl = env
    from xplgen import rodinia
    spec = rodinia.hotspot_spec(64, 64)
    ar = apps.Arena(spec)
    s = torch.cuda.Stream()
    run = apps.Run(None, s.cuda_stream, do_copies=True)
    apps.hotspot(run, ar, 64, 64, 2)
    assert run.r.n_diag == 0 and run.r.status == 0

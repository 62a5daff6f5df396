#!/usr/bin/env python
"""Where the instrumentation overhead of cfg2 and cfg3 goes.

  cfg2: per Rodinia-shaped program, instrumented vs twin: whole program, the
        kernels alone (events around each launch), the runtime kernels (live
        events, xpl_profile) and the host tracer time.
  cfg3: SW 16384^2 (32,767 per-diagonal epochs), instrumented vs twin, the
        runtime kernels, with and without the host segments / diagnoses.

  python tools/overhead_probe.py [--n 16384] [--skip-cfg2] [--skip-cfg3]
Prints one JSON object per part and a final one with everything.
"""
from __future__ import annotations

import argparse
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)


def cfg2(torch, apps, xpl, us):
    from xplgen import rodinia
    HOT, BACKPROP, BFS, NW = (1024, 1024, 20), (655360, 16), (1000000, 6), (2048, 10)
    hs, bs, fs, ns = (rodinia.hotspot_spec(*HOT[:2]), rodinia.backprop_spec(*BACKPROP),
                      rodinia.bfs_spec(*BFS), rodinia.nw_spec(NW[0]))
    ar = {k: apps.Arena(v) for k, v in (("hotspot", hs), ("backprop", bs), ("bfs", fs), ("nw", ns))}
    rodinia.fill_inputs("hotspot", ar["hotspot"].host_views(), 0x58504C01)
    rodinia.fill_inputs("backprop", ar["backprop"].host_views(), 0x58504C01)
    edges = rodinia.bfs_graph(BFS[0], BFS[1], 0x58504C02)
    nw_in = rodinia.nw_inputs(NW[0], NW[1], 0x58504C03)
    hc = torch.zeros(1, dtype=torch.int64, device="cuda")
    progs = {"hotspot": (apps.hotspot, HOT), "backprop": (apps.backprop, BACKPROP),
             "bfs": (apps.bfs, BFS + (hc,)), "nw": (apps.nw, NW + (nw_in["blosum"],))}
    res = {}
    with xpl.Context(pool_words=1 << 27, max_rows=256) as ctx:
        for rep in range(2):
            for name, (fn, args) in progs.items():
                r = {}
                for c, prof, tk in ((ctx, False, False), (None, False, False), (ctx, False, True),
                                    (None, False, True), (ctx, True, False)):
                    apps.bfs_prepare(ar["bfs"], BFS[0], BFS[1], edges, resident=True)
                    rodinia.nw_fill_host(ar["nw"].host_views(), ns, nw_in, NW[0])
                    hc.zero_()
                    torch.cuda.synchronize()
                    if prof:
                        ctx.profile(True)
                    rs = torch.cuda.ExternalStream(ctx.runtime_stream()) if c is not None else us
                    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
                    e0.record(rs)
                    us.wait_event(e0)
                    run = apps.Run(c, us.cuda_stream, do_copies=False, diag_each=True, params=(50, 0, 256),
                                   time_kernels=tk)
                    fn(run, ar[name], *args)
                    if c is not None:
                        ctx.join(rs.cuda_stream)
                    e1.record(rs)
                    e1.synchronize()
                    torch.cuda.synchronize()
                    key = ("instr" if c is not None else "twin") + ("_prof" if prof else "") + ("_k" if tk else "")
                    r[key] = {"ms": e0.elapsed_time(e1), "host_ms": run.r.host_ms, "epochs": run.r.epochs}
                    if tk:
                        r[key]["kernel_ms"] = run.r.kernel_ms
                    if prof:
                        p = ctx.profile_read(reset=True)
                        ctx.profile(False)
                        r[key]["runtime"] = {k: {"launches": v["launches"], "ms": v["ms"]}
                                             for k, v in p.items() if v["launches"]}
                r["slowdown"] = r["instr"]["ms"] / r["twin"]["ms"]
                r["kernel_slowdown"] = r["instr_k"]["kernel_ms"] / r["twin_k"]["kernel_ms"]
                res[name] = r
    return res


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--n", type=int, default=16384)
    ap.add_argument("--skip-cfg2", action="store_true")
    ap.add_argument("--skip-cfg3", action="store_true")
    a = ap.parse_args()
    import torch
    from paper_conf_ipps_pirkelbauerlvl20_b200 import apps, xpl
    from xplgen import sw
    n = m = a.n
    us = torch.cuda.Stream()
    out = {"n": n}
    if not a.skip_cfg2:
        out["cfg2"] = cfg2(torch, apps, xpl, us)
        print(json.dumps({"cfg2": out["cfg2"]}), flush=True)
    if a.skip_cfg3:
        print(json.dumps(out), flush=True)
        return
    spec = sw.sw_spec(n, m)
    ar = apps.Arena(spec)
    inp = sw.sw_inputs(n, m, 0x58504C04)

    def timed(ctx, tb, dg, prof=False):
        s = torch.cuda.ExternalStream(ctx.runtime_stream()) if ctx is not None else us
        torch.cuda.synchronize()
        if prof:
            ctx.profile(True)
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record(s)
        us.wait_event(e0)
        run = apps.Run(ctx, us.cuda_stream, params=(50, 0, 256))
        apps.sw(run, ar, n, m, 1, tb, dg, inp)
        if ctx is not None:
            ctx.join(s.cuda_stream)
        e1.record(s)
        e1.synchronize()
        torch.cuda.synchronize()
        r = {"ms": e0.elapsed_time(e1), "epochs": run.r.epochs, "host_ms": run.r.host_ms}
        if prof:
            p = ctx.profile_read(reset=True)
            ctx.profile(False)
            r["runtime"] = {k: {"launches": v["launches"], "ms": v["ms"]} for k, v in p.items() if v["launches"]}
        if ctx is not None:
            st = ctx.stats()
            r["stats"] = {k: st[k] for k in ("kernel_launches", "merge_segments", "range_segments", "folds")
                          if k in st}
        return r

    res3 = {}
    with xpl.Context(pool_words=1 << 29, max_rows=16) as ctx:
        for tb, dg in ((1024, 1024), (0, 0)):
            key = f"tb{tb}_dg{dg}"
            res3[key] = {"twin": timed(None, tb, dg), "instr": timed(ctx, tb, dg),
                        "instr_profiled": timed(ctx, tb, dg, prof=True)}
            o = res3[key]
            ep = o["instr"]["epochs"]
            o["us_per_diag_instr"] = 1e3 * o["instr"]["ms"] / ep
            o["us_per_diag_twin"] = 1e3 * o["twin"]["ms"] / ep
            o["overhead_us_per_diag"] = o["us_per_diag_instr"] - o["us_per_diag_twin"]
            print(json.dumps({key: o}), flush=True)
    out["cfg3"] = res3
    print(json.dumps(out), flush=True)


if __name__ == "__main__":
    main()

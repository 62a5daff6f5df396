#!/usr/bin/env python
"""Benchmark of the B200-native XPlacer recording + diagnosis hot path.

Headline workload = BASELINE.json configs[3] (cfg4, the largest single-GPU
config): the LULESH-shaped program, 100^3 mesh, 100 timesteps -- 50 managed
allocations + two temporaries allocated/freed per timestep, 19 instrumented
launches per timestep (every one a GPU epoch), host TimeIncrement segments
(traced), a diagnose after every timestep and after the final frees.  One
STEP = one whole run of that program through the C-ABI: every §8(a) row runs
(a1 register/free, a2 lookups, a3 device hooks, a4 epoch close, a5/a6 host
ingest + merge, a7 range apply of the host init ranges, a8 diagnose).

Metric (BASELINE.json): recorded accesses/s -- device hook calls + host tracer
calls -- per second of device time (CUDA events, runtime stream joined),
whole job; + diagnose GB/s; + the instrumented-kernel slowdown.
  value  the program's input (mesh topology) already in its managed arrays;
  e2e    the same, with the topology uploaded from pinned host memory inside
         the timed region (host-record staging and report copies are in both).
Also: the hook-path roofline in the step (instrumented kernels vs twins, events
on the kernels' stream), the runtime kernels (live events, profiled re-run),
the streaming microbenchmark (hook cost of a bandwidth-bound kernel), the
diagnose pass at cfg5 scale, the other configs (cfg1, cfg2, cfg3, cfg5), and
the oracle's rate on the host cores (cpu_baseline).

  python bench.py [--gpus N] [--steps K] [--warmup W] [--impl xpl|reference]
Under torchrun each rank runs its own instance (independent problems, weak
scaling, no data-path collective); rank 0 prints one JSON line.
"""
from __future__ import annotations

import argparse
import json
import os
import statistics
import subprocess
import sys
import tempfile
import time

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

S4, T4 = 100, 100  # cfg4: LULESH-shaped 100^3 x 100 timesteps
SEED4 = 0x58504C05
PARAMS = (50, 0, 256)  # threshold 50 %, whole-allocation blocks, min run 256 words (D16)
WORKLOAD = "cfg4: LULESH-shaped 100^3 mesh x 100 timesteps (50 managed allocations + 2 temporaries/timestep, " \
           "19 instrumented launches/timestep, diagnose every timestep)"


def workload(size, timesteps):
    if size == S4 and timesteps == T4:
        return WORKLOAD
    name = "cfg5: " if size == 250 else ""
    return (f"{name}LULESH-shaped {size}^3 mesh x {timesteps} timesteps (50 managed allocations + 2 "
            "temporaries/timestep, 19 instrumented launches/timestep, diagnose every timestep)")
METRIC = "recorded accesses/s (device hooks + host tracer) + diagnose GB/s; instrumented-kernel slowdown"
# Distinct shadow words per epoch summed over one cfg4 timestep (tools/lulesh_words.py 100): the
# unit count of the hook path's algorithmic bytes (1 B shadow read + <= 1 B written per word)
CFG4_WORDS_PER_TIMESTEP = 352_359_838
HOOK_BYTES_PER_WORD = 2
HOT = (1024, 1024, 20)
BACKPROP = (655360, 16)
BFS = (1000000, 6)
NW = (2048, 10)


def parse():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=3)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--impl", choices=["xpl", "reference"], default="xpl")
    ap.add_argument("--timesteps", type=int, default=T4, help="cfg4 timesteps per step (default 100)")
    ap.add_argument("--size", type=int, default=S4,
                    help="LULESH mesh edge (default 100 = cfg4; 250 = cfg5, e.g. sharded: --gpus 8 --size 250)")
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--no-other-configs", action="store_true")
    ap.add_argument("--step-only", action="store_true",
                    help="warm-up + timed steps only, no JSON line (for ncu captures of the step's kernels)")
    return ap.parse_args()


def peaks():
    try:
        with open(os.path.join(ROOT, "MEASURED_PEAKS.json")) as f:
            p = json.load(f)
        return float(p["hbm_gbs"]), "measured"
    except Exception:
        return 6650.0, "fallback"


class Clocks:
    """nvidia-smi sampling during the timed region (B200_PROFILING.md clocks line)."""

    def __init__(self, idx):
        self.f = tempfile.NamedTemporaryFile("w+", suffix=".csv", delete=False)
        q = ("index,clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.active,"
             "clocks_event_reasons.hw_slowdown,clocks_event_reasons.hw_thermal_slowdown,"
             "clocks_event_reasons.sw_thermal_slowdown,clocks_event_reasons.sw_power_cap")
        try:
            self.p = subprocess.Popen(["nvidia-smi", f"--id={idx}", f"--query-gpu={q}", "--format=csv,noheader,nounits",
                                       "-lms", "100"], stdout=self.f, stderr=subprocess.DEVNULL)
        except Exception:
            self.p = None
        self.off = 0

    def mark(self):
        """Start of the timed region: only samples written from here on count."""
        try:
            self.off = os.path.getsize(self.f.name)
        except OSError:
            self.off = 0

    def stop(self):
        if self.p is None:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["nvidia-smi unavailable"]}
        self.p.terminate()
        self.p.wait()
        self.f.flush()
        self.f.seek(self.off)
        sm, mx, reasons = [], None, set()
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        for line in self.f.read().splitlines():
            parts = [x.strip() for x in line.split(",")]
            if len(parts) < 9:
                continue
            try:
                sm.append(float(parts[1]))
                mx = float(parts[2])
            except ValueError:
                continue
            for n, v in zip(names, parts[5:9]):
                if v.lower().startswith("active"):
                    reasons.add(n)
        os.unlink(self.f.name)
        return {"sm_mhz": statistics.median(sm) if sm else None, "sm_max_mhz": mx,
                "reasons": sorted(reasons), "samples": len(sm)}


def cpu_baseline(seconds_budget=None):
    """The oracle as it stands, on a bounded sample of the cfg4 workload: timestep
    1 of the LULESH-shaped 100^3 program (host init + 19 kernel epochs + the host
    TimeIncrement + the diagnose), restricted to the events of `dom`, `dt_block`
    and the element array `e` (a word's record depends only on the events that
    touch it: the partitioned-by-allocation replay of SURVEY §8(d)); 1 thread."""
    import numpy as np
    from oracle import Oracle
    from xplgen import lulesh as L
    from xplgen.rodinia import layout
    spec = L.lulesh_spec(S4)
    addrs, _, _ = layout(spec, 0, 0, 1 << 40)
    topo = L.topology(S4, SEED4)
    win = {L.E: [(0, L.slot_bytes(S4, L.E) // 4)]}
    ops = list(L.lulesh_trace_iter(addrs, spec, S4, 1, topo, PARAMS, [((1 << 44), (1 << 44) + (1 << 33))],
                                   windows=win, reset=1, final=False))
    n_acc = sum(int(np.asarray(op[1]).size) for op in ops if op[0] in ("HB", "DB"))
    o = Oracle()
    t0 = time.perf_counter()
    done = 0
    for op in ops:
        o.op(op)
        if op[0] in ("HB", "DB"):
            done += int(np.asarray(op[1]).size)
        if seconds_budget is not None and time.perf_counter() - t0 > seconds_budget:
            break
    dt = time.perf_counter() - t0
    o.close()
    return {"value": done / dt, "unit": "accesses/s", "cores": 1, "kind": "oracle",
            "sample": f"cfg4 timestep 1 (LULESH-shaped 100^3: host init, 19 kernel epochs, TimeIncrement, "
                      f"diagnose) restricted to the events of dom, dt_block and e ({n_acc} accesses, "
                      f"{dt:.1f} s, 1 thread)"}


def _allsum(torch, dist, x):
    if not dist.is_available() or not dist.is_initialized():
        return x
    dev = "cuda" if dist.get_backend() == "nccl" else "cpu"
    t = torch.tensor([x], dtype=torch.float64, device=dev)
    dist.all_reduce(t, op=dist.ReduceOp.SUM)
    return float(t.item())


def make_comm(xpl, torch, dist, rank, world, local, backend):
    """The sharded context's collectives: libxpl.so's own NCCL communicator (its
    unique id broadcast over the process group), or gloo through torch."""
    if backend != "nccl":
        return xpl.TorchComm()

    def bcast(b):
        t = torch.tensor(list(b), dtype=torch.uint8, device="cuda")
        dist.broadcast(t, 0)
        return bytes(t.cpu().tolist())
    return xpl.NcclComm(rank, world, local, bcast)


def _allmax(torch, dist, x):
    if not dist.is_available() or not dist.is_initialized():
        return x
    dev = "cuda" if dist.get_backend() == "nccl" else "cpu"
    t = torch.tensor([x], dtype=torch.float64, device=dev)
    dist.all_reduce(t, op=dist.ReduceOp.MAX)
    return float(t.item())


def atomic_peaks(xpl, torch, reps=3):
    """32-bit atomic OR throughput of this B200 (in-repo microbenchmark, one op per
    distinct u32, coalesced): RED and ATOM over 1 GiB, RED over 32 MiB (L2), and
    every lane of a warp on one u32."""
    out = {}
    buf = torch.zeros(1 << 28, dtype=torch.int32, device="cuda")
    st = torch.cuda.current_stream()
    for name, n, mode in (("red_hbm", 1 << 28, 0), ("atom_hbm", 1 << 28, 1), ("red_l2", 1 << 23, 0),
                          ("red_same_word", 1 << 28, 2)):
        xpl.atomic_bench(buf.data_ptr(), n, mode, st.cuda_stream)
        torch.cuda.synchronize()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        k = reps if n >= (1 << 28) else reps * 16
        e0.record(st)
        for _ in range(k):
            xpl.atomic_bench(buf.data_ptr(), n, mode, st.cuda_stream)
        e1.record(st)
        e1.synchronize()
        out[name + "_per_s"] = k * n / (e0.elapsed_time(e1) / 1e3)
    del buf
    return out


def stream_microbench(xpl, torch, n=1 << 28, reps=5):
    """The hook path on a bandwidth-bound kernel with real data: y[i] = 2 x[i]
    over 1 GiB of 4-byte elements, every read traceR, every write traceW, in one
    epoch that first-touches every shadow word (the interval's REDs), against its
    twin -- with plain hooks (a row lookup per access) and through array handles
    (the lookup hoisted out of the loop).  Algorithmic bytes = 8 B of data + 2 x 2 B
    of shadow per element (1 B read + 1 B written per word on
    first touch); slowdown floor 1.5."""
    peak, _ = peaks()
    st = torch.cuda.Stream()
    s = st.cuda_stream
    x = torch.ones(n, dtype=torch.int32, device="cuda")
    y = torch.empty_like(x)

    def ev(fn):
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record(st)
        fn()
        e1.record(st)
        e1.synchronize()
        return e0.elapsed_time(e1)
    twin = min(ev(lambda: xpl.stream_kernel(x.data_ptr(), y.data_ptr(), n, 4, 0, s)) for _ in range(reps))
    data, shadow = 8 * n, 4 * n
    out = {"n": n, "elem_bytes": 4, "twin_ms": twin, "slowdown_floor": (data + shadow) / data, "peak_gbs": peak,
           "twin_gbs": data / (twin / 1e3) / 1e9}
    with xpl.Context(pool_words=2 * n + (1 << 20), max_rows=16) as ctx:
        ctx.register(x.data_ptr(), 4 * n, xpl.ALLOC_DEVICE)
        ctx.register(y.data_ptr(), 4 * n, xpl.ALLOC_DEVICE)
        for mode, name in ((1, "plain"), (2, "handles")):
            first, fold = [], []
            for _ in range(reps):
                ctx.diagnose(*PARAMS, reset=True)  # a fresh interval: every shadow word is first-touched again
                torch.cuda.synchronize()
                ctx.kernel_begin(s)
                e0, e1, e2 = (torch.cuda.Event(enable_timing=True) for _ in range(3))
                e0.record(st)
                xpl.stream_kernel(x.data_ptr(), y.data_ptr(), n, 4, mode, s)
                e1.record(st)
                ctx.kernel_end(s)
                ctx.join(s)
                e2.record(st)
                e2.synchronize()
                first.append(e0.elapsed_time(e1))
                fold.append(e1.elapsed_time(e2))
            ms = min(first)
            out[name] = {"instr_ms": ms, "epoch_close_ms": min(fold), "slowdown": ms / twin,
                         "achieved_gbs": (data + shadow) / (ms / 1e3) / 1e9,
                         "frac": (data + shadow) / (ms / 1e3) / 1e9 / peak,
                         "hooked_accesses_per_s": 2 * n / (ms / 1e3)}
    del x, y
    torch.cuda.empty_cache()
    return out


def diag_at_scale(xpl, torch, words=1 << 31, reps=3):
    """The diagnose pass over a cfg5-sized shadow (2^31 words = 2 GiB) with a mixed
    content (per 4096-word block: untouched / all read / all written / per-word
    random R, W, RW; first half CPU-written); live CUDA events (xpl_profile)."""
    ctx = xpl.Context(pool_words=words + (1 << 16), max_rows=16)
    base = 1 << 44  # synthetic address range: hooks only use addresses
    ctx.register(base, 4 * words, xpl.ALLOC_DEVICE)
    ctx.record_copy(base, 0x1000, 2 * words, xpl.COPY_H2D)
    st = torch.cuda.current_stream()
    s = st.cuda_stream
    ctx.sync()
    torch.cuda.synchronize()
    ctx.profile(True)
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record(st)
    ctx.kernel_begin(s)
    ctx.touch(base, words, 7, s, 0)
    ctx.kernel_end(s)
    ctx.join(s)
    e1.record(st)
    e1.synchronize()
    rec_ms = e0.elapsed_time(e1)
    pf = ctx.profile_read(reset=True)["fold"]
    ctx.sync()
    torch.cuda.synchronize()
    for _ in range(reps):
        ctx.diagnose(*PARAMS, reset=False)
    p0 = ctx.profile_read(reset=True)
    ctx.page_summary(1024)
    pv = []
    for _ in range(reps):
        t0 = time.perf_counter()
        ctx.page_summary(1024)
        pv.append((time.perf_counter() - t0) * 1e3)
    rep = ctx.diagnose(*PARAMS, reset=True)
    p1 = ctx.profile_read(reset=True)
    ctx.profile(False)
    ctx.close()
    n_dev = rep[0]["gpu_acc"]
    out = {"record_touch": {"device_accesses": n_dev, "ms": rec_ms, "accesses_per_s": n_dev / (rec_ms / 1e3),
                            "fold_ms": pf["ms"],
                            "fold_gbs": pf["bytes"] / (pf["ms"] / 1e3) / 1e9 if pf["ms"] else None,
                            "note": "synthetic touch kernel (per-lane access kinds, hooks only) + epoch close"},
           "page_view": {"words": words, "page_words": 1024, "whole_call_ms": min(pv),
                         "kernel_ms": p1["pages"]["ms"] / max(1, p1["pages"]["launches"]),
                         "gbs": (p1["pages"]["bytes"] / (p1["pages"]["ms"] / 1e3) / 1e9) if p1["pages"]["ms"] else None}}
    for name, p in (("no_reset", p0), ("reset", p1)):
        d = p["diag_tile"]
        ms = d["ms"] / d["launches"]
        out[name] = {"words": words, "ms": ms, "gbs": d["bytes"] / d["launches"] / (ms / 1e3) / 1e9,
                     "bytes_per_launch": d["bytes"] / d["launches"],
                     "whole_call_ms": p["diagnose"]["ms"] / p["diagnose"]["launches"]}
    return out


class Cfg4:
    """The cfg4 program's arrays, input and runs."""

    def __init__(self, torch, apps, timesteps, rank=0, world=1, size=S4):
        from xplgen import lulesh as L
        self.torch, self.apps, self.T, self.S = torch, apps, timesteps, size
        self.rank, self.world = rank, world  # world > 1: the sharded program (this rank's slab)
        self.spec = L.lulesh_spec(size)
        self.ar = apps.Arena(self.spec)
        self.topo = L.topology(size, SEED4)
        self.host_topo = apps.lulesh_topology_host(self.topo)
        self.hc = torch.zeros(1, dtype=torch.int64, device="cuda")
        self.us = torch.cuda.Stream()
        self.input_bytes = sum(t.numel() * t.element_size() for t in self.host_topo.values())

    def prepare(self, resident=True):
        self.hc.zero_()
        if resident:
            self.apps.lulesh_prepare(self.ar, self.S, self.topo)

    def run(self, ctx, upload=False, time_kernels=False, params=PARAMS):
        """One step: the whole program.  upload: the topology H2D first (e2e)."""
        if upload:
            self.apps.lulesh_upload(self.ar, self.host_topo, self.us.cuda_stream)
        run = self.apps.Run(ctx, self.us.cuda_stream, params=params, out_cap=64 * (self.T + 2),
                            time_kernels=time_kernels, rank=self.rank, world=self.world)
        self.apps.lulesh(run, self.ar, self.S, self.T, self.hc)
        return run


def timed_steps(torch, c4, ctx, steps, upload=False, flush=None):
    """Device time of `steps` whole-program steps (events on the runtime stream,
    which is joined to the program's stream before the end event)."""
    total, acc = 0.0, []
    rs = torch.cuda.ExternalStream(ctx.runtime_stream()) if ctx is not None else c4.us
    for _ in range(steps):
        c4.prepare(resident=not upload)
        if flush is not None:
            flush.random_(0, 255)  # > L2: flushed between steps (untimed)
        torch.cuda.synchronize()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record(rs)
        if ctx is not None:
            c4.us.wait_event(e0)
        run = c4.run(ctx, upload=upload)
        if ctx is not None:
            ctx.join(rs.cuda_stream)
        else:
            pass
        e1.record(rs if ctx is not None else c4.us)
        e1.synchronize()
        torch.cuda.synchronize()
        total += e0.elapsed_time(e1)
        acc.append((int(c4.hc.item()), run.r.host_accesses, run.r.epochs, run.r.n_diag, run.r.n_out))
    c4.last_reports = run.reports() if ctx is not None else None
    return total, acc


def rodinia_step(xpl, apps, torch):
    """configs[1] (round 1's headline): hotspot + backprop + bfs + nw, one step, app
    data resident, instrumented and as twin (events around each program)."""
    from xplgen import rodinia
    hs, bs, fs, ns = (rodinia.hotspot_spec(HOT[0], HOT[1]), rodinia.backprop_spec(*BACKPROP),
                      rodinia.bfs_spec(*BFS), rodinia.nw_spec(NW[0]))
    ar = {k: apps.Arena(v) for k, v in (("h", hs), ("b", bs), ("f", fs), ("n", ns))}
    rodinia.fill_inputs("hotspot", ar["h"].host_views(), 0x58504C01)
    rodinia.fill_inputs("backprop", ar["b"].host_views(), 0x58504C01)
    edges = rodinia.bfs_graph(BFS[0], BFS[1], 0x58504C02)
    nw_in = rodinia.nw_inputs(NW[0], NW[1], 0x58504C03)
    hc = torch.zeros(1, dtype=torch.int64, device="cuda")
    us = torch.cuda.Stream()
    res = {}
    with xpl.Context(pool_words=1 << 27, max_rows=256) as ctx:
        for rep in range(2):
            for c in (ctx, None):
                apps.bfs_prepare(ar["f"], BFS[0], BFS[1], edges, resident=True)
                rodinia.nw_fill_host(ar["n"].host_views(), ns, nw_in, NW[0])
                hc.zero_()
                torch.cuda.synchronize()
                rs = torch.cuda.ExternalStream(ctx.runtime_stream()) if c is not None else us
                e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
                e0.record(rs)
                us.wait_event(e0)
                n_acc = 0
                for fn, a, args in ((apps.hotspot, ar["h"], HOT), (apps.backprop, ar["b"], BACKPROP),
                                    (apps.bfs, ar["f"], BFS + (hc,)), (apps.nw, ar["n"], NW + (nw_in["blosum"],))):
                    run = apps.Run(c, us.cuda_stream, do_copies=False, diag_each=True, params=PARAMS)
                    fn(run, a, *args)
                    n_acc += run.r.dev_accesses + run.r.host_accesses + run.r.copy_words
                if c is not None:
                    ctx.join(rs.cuda_stream)
                e1.record(rs)
                e1.synchronize()
                torch.cuda.synchronize()
                n_acc += int(hc.item())
                res["instr" if c is not None else "twin"] = (e0.elapsed_time(e1), n_acc)
    ms, acc = res["instr"]
    return {"workload": "cfg2 rodinia: hotspot 1024x1024x20 + backprop 640Kx16 + bfs 1Mx6 + nw 2048x2048 "
                        "(data resident, diagnose every iteration)",
            "ms": ms, "accesses": acc, "accesses_per_s": acc / (ms / 1e3), "twin_ms": res["twin"][0],
            "slowdown": ms / res["twin"][0]}


def other_configs(xpl, apps, torch, lulesh250_steps=100):
    """cfg1 SW-128 (one launch; one cooperative launch with a device-side split per
    diagonal), cfg2 Rodinia, cfg3 SW-16K (32,767 per-diagonal epochs), cfg5
    LULESH-shaped 250^3 x 100 timesteps on one GPU -- instrumented and as twin."""
    from xplgen import lulesh as L
    from xplgen import sw
    out = {}
    us = torch.cuda.Stream()

    def timed_run(ctx, fn):
        s = torch.cuda.ExternalStream(ctx.runtime_stream()) if ctx is not None else us
        torch.cuda.synchronize()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record(s)
        us.wait_event(e0)
        run = fn(ctx)
        if ctx is not None:
            ctx.join(s.cuda_stream)
        e1.record(s)
        e1.synchronize()
        torch.cuda.synchronize()
        return e0.elapsed_time(e1), run

    for name, (n, m, per_diag, tb, dg, pool) in {
            "cfg1_sw128": (128, 128, 0, 0, 0, 1 << 20),
            "cfg1_sw128_split": (128, 128, 2, 0, 0, 1 << 20),
            "cfg3_sw16k": (16384, 16384, 1, 1024, 1024, 1 << 29)}.items():
        spec = sw.sw_spec(n, m)
        ar = apps.Arena(spec)
        inp = sw.sw_inputs(n, m, 0x58504C04)
        res = {}
        with xpl.Context(pool_words=pool, max_rows=16) as ctx:
            # (a first, untimed-in-effect twin run populates the fresh managed
            # arena's host pages -- the program zeroes H on the host -- so that
            # cost falls on neither timed run; its result is overwritten)
            for c in (None, ctx, None):
                def fn(c):
                    run = apps.Run(c, us.cuda_stream, params=PARAMS)
                    apps.sw(run, ar, n, m, per_diag, tb, dg, inp)
                    return run
                ms, run = timed_run(c, fn)
                res["instr" if c is not None else "twin"] = (ms, run.r.dev_accesses + run.r.host_accesses,
                                                            run.r.epochs, run.r.n_diag)
        acc = res["instr"][1]
        out[name] = {"workload": f"Smith-Waterman {n}x{m}, managed, "
                                 + ["one launch", "per-diagonal launches",
                                    "one cooperative launch, device-side epoch split per diagonal"][per_diag],
                     "ms": res["instr"][0], "accesses": acc, "accesses_per_s": acc / (res["instr"][0] / 1e3),
                     "epochs": res["instr"][2], "diagnoses": res["instr"][3], "twin_ms": res["twin"][0],
                     "slowdown": res["instr"][0] / res["twin"][0]}
        del ar
    out["cfg2_rodinia"] = rodinia_step(xpl, apps, torch)
    if lulesh250_steps:
        s_edge, steps = 250, lulesh250_steps
        spec = L.lulesh_spec(s_edge)
        ar = apps.Arena(spec)
        topo = L.topology(s_edge, SEED4)
        hc = torch.zeros(1, dtype=torch.int64, device="cuda")
        res = {}
        with xpl.Context(pool_words=2_500_000_000, max_rows=64) as ctx:
            for c in (ctx, None):
                apps.lulesh_prepare(ar, s_edge, topo)
                hc.zero_()

                def fn(c):
                    run = apps.Run(c, us.cuda_stream, params=PARAMS, out_cap=64 * (steps + 2))
                    apps.lulesh(run, ar, s_edge, steps, hc)
                    return run
                ms, run = timed_run(c, fn)
                res["instr" if c is not None else "twin"] = (ms, int(hc.item()) + run.r.host_accesses,
                                                            run.r.epochs, run.r.n_diag, run.r.host_ms)
        del ar, topo
        acc = res["instr"][1]
        out["cfg5_lulesh250"] = {
            "workload": f"LULESH-shaped 250^3 x {steps} timesteps on one GPU, 50 managed allocations + "
                        "2 temporaries/timestep, 19 launches/timestep",
            "ms": res["instr"][0], "accesses": acc, "accesses_per_s": acc / (res["instr"][0] / 1e3),
            "epochs": res["instr"][2], "diagnoses": res["instr"][3], "host_ms": res["instr"][4],
            "twin_ms": res["twin"][0], "slowdown": res["instr"][0] / res["twin"][0]}
    return out


def hook_roofline(args, hook_ms, k_instr, k_twin, ms_step, prof, peak, peak_src, hook_unpaired=None):
    hook_bytes = HOOK_BYTES_PER_WORD * CFG4_WORDS_PER_TIMESTEP
    # (the distinct-word count is the 100^3 mesh's; other sizes report the time only)
    ach = hook_bytes / (hook_ms / 1e3) / 1e9 if hook_ms > 0 and args.size == S4 else None
    return {"kernel": "device hooks (a3), inlined in the 19 instrumented launches of each timestep",
            "bound": "hbm", "achieved": ach, "peak": peak, "unit": "GB/s",
            "frac": (ach / peak) if ach else None, "traffic": None, "peak_source": peak_src,
            "algorithmic_bytes_per_timestep": hook_bytes,
            "algorithmic_model": "2 B (shadow byte read + written) per distinct word per epoch; "
                                 f"{CFG4_WORDS_PER_TIMESTEP} distinct words per timestep (tools/lulesh_words.py)",
            "hook_ms_per_timestep": hook_ms,
            "timing": "CUDA events on the program's stream around each of the 1900 launches of a measurement "
                      "run in which every instrumented launch is paired with its twin (twin first on odd "
                      "launches, second on even; L2 flushed before each); per launch position the mean over "
                      "the two orders of the "
                      "median over the timesteps of instrumented minus twin, summed over the 19 positions",
            "hook_ms_per_timestep_unpaired": hook_unpaired,
            "share_of_step": hook_ms * args.timesteps / ms_step,
            "kernels_ms_per_step": {"instrumented": k_instr, "twin": k_twin},
            "runtime_kernels_ms_per_step": {k: v["ms"] for k, v in prof.items() if k != "diagnose"}}


def sharded_tail(args, torch, dist, apps, xpl, rank, world, value, ms_max, per_step, epochs, n_diag, e2e,
                 launches, clocks, twin_ms, k_instr, k_twin, prof, sharded_reports, peak, peak_src, backend,
                 hook_med):
    """N > 1: the line of the sharded cfg4 program; rank 0 also runs the 1-GPU
    program and checks every report (but `base`) is identical."""
    identical = None
    if rank == 0:
        c1 = Cfg4(torch, apps, args.timesteps, size=args.size)
        pool = 1 << 28 if args.size <= S4 else 2_500_000_000
        with xpl.Context(device=torch.cuda.current_device(), pool_words=pool, max_rows=64) as ctx1:
            c1.prepare()
            one = c1.run(ctx1).reports()
        # (ids continue across the context's runs, bases are each program's own)
        strip = lambda ds: [[{f: v for f, v in r.items() if f not in ("base", "id")} for r in d] for d in ds]
        a, b = strip(one), strip(sharded_reports)
        identical = a == b
        if not identical:  # the first difference, for the record
            for k, (da, db) in enumerate(zip(a, b)):
                if da != db:
                    for i, (ra, rb) in enumerate(zip(da, db)):
                        if ra != rb:
                            first_diff = {"diagnose": k, "row": i,
                                          "fields": {f: (ra[f], rb[f]) for f in ra if ra[f] != rb[f]}}
                            break
                    else:
                        first_diff = {"diagnose": k, "rows": (len(da), len(db))}
                    break
            else:
                first_diff = {"diagnoses": (len(a), len(b))}
            print(json.dumps({"identity_first_difference": first_diff}), file=sys.stderr, flush=True)
    roof = hook_roofline(args, hook_med, k_instr, k_twin, ms_max / args.steps, prof, peak, peak_src)
    line = {"metric": METRIC, "value": value, "unit": "accesses/s", "n_gpus": world, "steps": args.steps,
            "warmup": args.warmup, "ms_per_step": ms_max / args.steps, "higher_is_better": True,
            "scaling": "strong", "vs_baseline": None, "dtype": "u8", "data": "synthetic",
            "config": {"workload": workload(args.size, args.timesteps) + f", sharded over {world} GPUs (one logical program: each rank "
                                              "its slab of elements/nodes; shadow partitioned by word, host "
                                              "records routed all-to-all, remote hook atomics, partials combined)",
                       "timesteps": args.timesteps, "accesses_per_step": per_step, "epochs_per_step": epochs,
                       "diagnoses_per_step": n_diag, "parallelism": f"sharded x{world}",
                       "collectives": "NCCL (libxpl.so xpl_comm_nccl)" if backend == "nccl" else backend,
                       "l2": "flushed between steps (256 MB write, untimed)"},
            "roofline": roof, "e2e": e2e, "gpu_launches": int(launches), "clocks": clocks,
            "summary": {"accesses_per_s": value, "e2e_accesses_per_s": e2e["value"],
                        "reports_identical_to_1gpu": identical,
                        "slowdown_whole_program": (ms_max / args.steps) / (twin_ms / args.steps),
                        "slowdown_kernels": k_instr / k_twin if k_twin else None}}
    if rank == 0:
        print(json.dumps(line), flush=True)
    dist.barrier()
    dist.destroy_process_group()


def reference_main(args):
    rank = int(os.environ.get("RANK", "0"))
    if rank != 0:
        return
    for _ in range(args.warmup):  # untimed warm-up samples (short)
        cpu_baseline(seconds_budget=1.0)
    steps = [cpu_baseline() for _ in range(max(1, args.steps))]
    v = statistics.median(s["value"] for s in steps)
    line = {"impl": "reference", "metric": METRIC, "value": v, "unit": "accesses/s",
            "n_gpus": args.gpus, "steps": args.steps, "warmup": args.warmup,
            "higher_is_better": True, "scaling": "weak", "vs_baseline": None, "dtype": "u8",
            "data": "synthetic", "config": {"workload": WORKLOAD},
            "cpu_baseline": {"value": v, "unit": "accesses/s", "cores": 1, "kind": "oracle",
                             "sample": steps[0]["sample"]},
            "e2e": {"value": v, "unit": "accesses/s", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}}
    print(json.dumps(line), flush=True)


def main():
    args = parse()
    if args.impl == "reference":
        return reference_main(args)
    import torch
    import torch.distributed as dist

    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0")) % max(1, torch.cuda.device_count())
    torch.cuda.set_device(local)
    backend = os.environ.get("XPL_DIST_BACKEND", "nccl")  # gloo: the N>1 logic on one GPU
    if world > 1:
        if backend == "nccl":
            dist.init_process_group("nccl", device_id=torch.device("cuda", local))
        else:
            dist.init_process_group(backend)

    from paper_conf_ipps_pirkelbauerlvl20_b200 import apps, xpl

    # N > 1: the cfg4 program sharded over the ranks (each its slab; one logical
    # program, shadow partitioned by word over the GPUs, xpl.h sharded mode)
    c4 = Cfg4(torch, apps, args.timesteps, rank, world, args.size)
    comm = make_comm(xpl, torch, dist, rank, world, local, backend) if world > 1 else None
    pool = 1 << 28 if args.size <= S4 else 2_500_000_000  # (cfg5: 2.3e9 shadow words per timestep)
    ctx = xpl.Context(device=local, pool_words=pool, max_rows=256, comm=comm)
    flush_buf = torch.empty(256 << 20, dtype=torch.uint8, device="cuda")  # > 126 MB L2

    clk = Clocks(local)
    for _ in range(args.warmup):
        c4.prepare()
        c4.run(ctx)
    torch.cuda.synchronize()

    # --- value: device-timed, program input resident -------------------------
    st0 = ctx.stats()
    if world > 1:
        dist.barrier()
    torch.cuda.synchronize()
    clk.mark()
    ms_total, acc = timed_steps(torch, c4, ctx, args.steps, flush=flush_buf)
    clocks = clk.stop()
    st1 = ctx.stats()
    hooks, host_acc, epochs, n_diag, n_rows = acc[-1]
    sharded_reports = c4.last_reports if world > 1 else None  # (the last timed step's reports)
    per_step = int(_allsum(torch, dist, hooks + host_acc))  # the logical program's accesses
    ms_max = _allmax(torch, dist, ms_total)
    value = per_step * args.steps / (ms_max / 1e3)
    launches = (st1["kernel_launches"] - st0["kernel_launches"]) + epochs * args.steps
    if args.step_only:
        ctx.close()
        return

    # --- e2e: the topology uploaded from pinned host memory inside the region ---
    st0 = ctx.stats()
    if world > 1:
        dist.barrier()
    e2e_ms, _ = timed_steps(torch, c4, ctx, args.steps, upload=True, flush=flush_buf)
    st1 = ctx.stats()
    e2e_ms = _allmax(torch, dist, e2e_ms)
    rec_bytes = 8 * (st1["host_records_packed"] - st0["host_records_packed"]) // args.steps
    e2e = {"value": per_step * args.steps / (e2e_ms / 1e3), "unit": "accesses/s",
           "h2d_bytes_per_step": c4.input_bytes + rec_bytes,
           "d2h_bytes_per_step": xpl.REPORT_BYTES * n_rows}

    # --- uninstrumented twin (whole-program slowdown) ---------------------------
    twin_ms, _ = timed_steps(torch, c4, None, args.steps, flush=flush_buf)
    twin_ms = _allmax(torch, dist, twin_ms)

    # --- hook path: kernels alone, instrumented vs twin, events on their stream --
    c4.prepare()
    ri = c4.run(ctx, time_kernels=True)
    c4.prepare()
    rt = c4.run(None, time_kernels=True)
    torch.cuda.synchronize()
    k_instr, k_twin = _allmax(torch, dist, ri.r.kernel_ms), _allmax(torch, dist, rt.r.kernel_ms)
    # the hooks' cost per timestep: per launch position (19 per timestep), the median
    # over the timesteps of instrumented minus twin (the application's own unified-
    # memory faults vary launch to launch; the median per position is robust to them)
    import numpy as np
    nl = 19 * args.timesteps
    ai = np.array(ri.kernel_each[:nl]).reshape(args.timesteps, 19)
    at = np.array(rt.kernel_each[:nl]).reshape(args.timesteps, 19)
    hook_unpaired = float(np.sum(np.median(ai, axis=0) - np.median(at, axis=0)))
    # paired (the headline's hook cost): one measurement run of the instrumented
    # program in which every launch also runs its twin right before or after it
    # (alternating), both timed, each after an L2 flush -- per launch position,
    # the mean of the two orders' medians of (instrumented - twin): the
    # unified-memory faults the first of a pair pays cancel between the orders
    c4.prepare()
    rp = c4.run(ctx, time_kernels=2)
    torch.cuda.synchronize()
    ap = np.array(rp.kernel_each[:2 * nl]).reshape(args.timesteps, 19, 2)
    twin_first = (np.arange(nl).reshape(args.timesteps, 19) & 1).astype(bool)
    d = np.where(twin_first, ap[:, :, 1] - ap[:, :, 0], ap[:, :, 0] - ap[:, :, 1])  # instrumented - twin
    hook_med = float(sum(0.5 * (np.median(d[twin_first[:, p], p]) + np.median(d[~twin_first[:, p], p]))
                         for p in range(19)))
    hook_med = _allmax(torch, dist, hook_med)
    hook_unpaired = _allmax(torch, dist, hook_unpaired)

    # --- runtime kernels: a profiled re-run (events around every runtime kernel) --
    ctx.profile(True)
    ms_prof, _ = timed_steps(torch, c4, ctx, 1, flush=flush_buf)
    prof = ctx.profile_read(reset=True)
    ctx.profile(False)
    ctx.close()
    if comm is not None and hasattr(comm, "close"):
        comm.close()
    del flush_buf
    torch.cuda.empty_cache()

    peak, peak_src = peaks()
    if world > 1:
        return sharded_tail(args, torch, dist, apps, xpl, rank, world, value, ms_max, per_step, epochs, n_diag,
                            e2e, launches, clocks, twin_ms, k_instr, k_twin, prof, sharded_reports, peak, peak_src,
                            backend, hook_med)

    # --- microbenchmarks and the other configs --------------------------------
    smb = stream_microbench(xpl, torch)
    at_scale = diag_at_scale(xpl, torch)
    atom = atomic_peaks(xpl, torch)
    others = other_configs(xpl, apps, torch) if not args.no_other_configs else None

    # --- roofline: the dominant cost of our path in the step = the device hooks --
    roof = hook_roofline(args, hook_med, k_instr, k_twin, ms_total / args.steps, prof, peak, peak_src,
                         hook_unpaired)
    rt_ms = roof["runtime_kernels_ms_per_step"]
    dg = prof["diag_tile"]
    line = {
        "metric": METRIC,
        "value": value, "unit": "accesses/s", "n_gpus": world, "steps": args.steps, "warmup": args.warmup,
        "ms_per_step": ms_max / args.steps, "higher_is_better": True, "scaling": "weak",
        "vs_baseline": None, "dtype": "u8", "data": "synthetic",
        "config": {"workload": workload(args.size, args.timesteps), "timesteps": args.timesteps,
                   "accesses_per_step": per_step,
                   "device_accesses": hooks, "host_accesses": host_acc, "epochs_per_step": epochs,
                   "diagnoses_per_step": n_diag,
                   "diag_params": {"threshold_pct": PARAMS[0], "block_words": PARAMS[1], "min_run": PARAMS[2]},
                   "l2": "flushed between steps (256 MB write, untimed)", "parallelism": f"replicas x{world}"},
        "roofline": roof,
        "e2e": e2e, "gpu_launches": int(launches), "clocks": clocks,
        "breakdown_ms_per_step": {"instrumented_kernels": k_instr, "twin_kernels": k_twin,
                                  "host_tracer_and_program": ri.r.host_ms,
                                  "runtime_kernels": sum(v for k, v in rt_ms.items() if k != "diag_tile"),
                                  "profiled_step_ms": ms_prof},
        "runtime_kernels": {k: {"launches": v["launches"], "ms_per_step": v["ms"],
                                "gbs": (v["bytes"] / (v["ms"] / 1e3) / 1e9) if v["ms"] else None}
                            for k, v in prof.items()},
        "stream_microbench": smb,
        "diagnose_at_scale": dict(at_scale, peak_gbs=peak, frac_reset=at_scale["reset"]["gbs"] / peak,
                                  frac_no_reset=at_scale["no_reset"]["gbs"] / peak),
        "atomic_microbench": atom,
        "other_configs": others,
    }
    if rank == 0 and world == 1 and not args.no_cpu_baseline:
        line["cpu_baseline"] = cpu_baseline()
    # the metric's numbers last, so a truncated tail of the line still carries them
    line["summary"] = {
        "accesses_per_s": value, "e2e_accesses_per_s": e2e["value"],
        "diagnose_gbs": at_scale["reset"]["gbs"], "diagnose_frac": at_scale["reset"]["gbs"] / peak,
        "diagnose_gbs_no_reset": at_scale["no_reset"]["gbs"],
        "diagnose_gbs_in_step": (dg["bytes"] / (dg["ms"] / 1e3) / 1e9) if dg["ms"] else None,
        "hook_frac": roof["frac"],  # (paired, isolated: see roofline.timing)
        "hook_ms_per_timestep": roof["hook_ms_per_timestep"],
        "hook_ms_per_timestep_unpaired": roof.get("hook_ms_per_timestep_unpaired"),
        "stream_hook_frac": smb["plain"]["frac"],
        "stream_slowdown": smb["plain"]["slowdown"], "stream_handles_slowdown": smb["handles"]["slowdown"],
        "stream_handles_frac": smb["handles"]["frac"],
        "slowdown_whole_program": ms_total / twin_ms, "slowdown_kernels": k_instr / k_twin,
        "paper_slowdown_context": "Table III P:L431-443: 5x-20x, avg ~15x (Intel E5-2695 v4 + Pascal, CUDA 9.2)"}
    if rank == 0:
        print(json.dumps(line), flush=True)
    if world > 1:
        dist.destroy_process_group()


if __name__ == "__main__":
    main()

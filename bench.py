#!/usr/bin/env python
"""Benchmark of the B200-native XPlacer recording + diagnosis hot path.

One STEP = one pass of the whole hot path over the
configs[1] workload of BASELINE.json: the Rodinia-shaped instrumented programs
(hotspot 1024x1024 x 20 iterations, backprop 640K x 16, bfs 1M nodes x 6, nw
2048 x 2048) run end to end through
the C-ABI -- registration, host-tracer batches (merge), traced transfers
(range apply), instrumented kernels (device hooks) in GPU epochs (fold), and a
diagnose after every iteration and at the end (diagnose kernels), then frees.

Metric (BASELINE.json): recorded accesses/s -- host tracer calls + device hook
calls + transferred words -- per second of device time, whole job (all ranks).
value: data of the apps resident in HBM (their cudaMemcpy not performed).
e2e:   the same programs with their real host<->device copies (pinned host
       buffers) inside the timed region.
Also reported: the diagnose-kernel bandwidth, kernel-only and whole-program
slowdown vs the uninstrumented twins, the roofline of the dominant runtime
kernel (live CUDA-event timing on the runtime stream), and the oracle's rate
on the host cores (cpu_baseline).

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

HOT = (1024, 1024, 20)
BACKPROP = (655360, 16)
BFS = (1000000, 6)
NW = (2048, 10)
PARAMS = (50, 0, 256)  # threshold 50 %, whole-allocation blocks, min run 256 words
WORKLOAD = "rodinia: hotspot 1024x1024x20 + backprop 640Kx16 + bfs 1Mx6 + nw 2048x2048"
METRIC = "recorded accesses/s (host tracer + device hooks + transferred words)"


def parse():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=5)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--impl", choices=["xpl", "reference"], default="xpl")
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
        """Start of the timed region: only samples written from here on count.  (The
        sampler is started before the warm-up, so nvidia-smi's own start-up -- NVML
        init, a cold exec -- does not land in the timed host-bound step.)"""
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
    """The oracle as it stands, on a bounded sample of the same workload:
    hotspot 1024x1024 (first iterations) replayed event by event (~8-15 s on one
    core).  seconds_budget: stop early (untimed warm-up only -- the count would
    then not match the work done)."""
    from oracle import Oracle
    from xplgen import rodinia
    rows, cols, _ = HOT
    spec = rodinia.hotspot_spec(rows, cols)
    addrs, _, _ = rodinia.layout(spec, 1 << 40, 1 << 44)
    iters = 2
    ops = rodinia.hotspot_trace(addrs, spec, rows, cols, iters, True, PARAMS)
    n_acc = 2 * rows * cols + iters * rodinia.hotspot_accesses(rows, cols)
    o = Oracle()
    t0 = time.perf_counter()
    for op in ops:
        if op[0] == "X" and op[1] == 1:  # stop before the final transfer: sample = init + iterations
            break
        o.op(op)
        if seconds_budget is not None and time.perf_counter() - t0 > seconds_budget:
            break
    dt = time.perf_counter() - t0
    o.close()
    n_acc += 2 * rows * cols  # the two H2D transfers
    return {"value": n_acc / dt, "unit": "accesses/s", "cores": 1, "kind": "oracle",
            "sample": f"hotspot {rows}x{cols}: host init + 2 H2D + {iters} instrumented iterations "
                      f"with a diagnose after each ({n_acc} accesses, {dt:.1f} s, 1 thread)"}


def diag_sharded(xpl, torch, dist, rank, world, words=1 << 31, reps=3, check_1gpu=True):
    """Address-range sharding of the cfg5-sized shadow over the ranks:
    rank r holds words [r*W/N, (r+1)*W/N) of one logical allocation, records its
    part (H2D of the logical first half + the instrumented touch kernel with the
    logical pattern), diagnoses into partials; the partials are all-gathered and
    combined on every rank.  Timed: partial diagnose + exchange + combine, max over
    ranks.  Rank 0 also diagnoses the unsharded allocation and checks the combined
    report is byte-identical (shard-count invariance)."""
    import time
    chunk = -(-words // world)
    goff = rank * chunk
    n = max(0, min(words, goff + chunk) - goff)
    base = 1 << 44
    ctx = xpl.Context(pool_words=n + (1 << 16), max_rows=16)
    s = torch.cuda.current_stream().cuda_stream
    ctx.register_piece(base + 4 * goff, 4 * n, xpl.ALLOC_DEVICE, 0, goff, 4 * words)
    h0, h1 = goff, min(goff + n, words // 2)
    if h1 > h0:
        ctx.record_copy(base + 4 * h0, 0x1000, 4 * (h1 - h0), xpl.COPY_H2D)
    ctx.kernel_begin(s)
    ctx.touch(base + 4 * goff, n, 7, s, goff)
    ctx.kernel_end(s)
    ctx.sync()
    ms = []
    got = None
    for _ in range(reps):
        dist.barrier()
        torch.cuda.synchronize()
        t0 = time.perf_counter()
        blob = ctx.diagnose_partials(50, 0, 256, reset=False)
        # every rank holds a piece of every logical allocation: equal-size partials,
        # one all_gather over the process group's backend (NCCL over NVLink on GPUs)
        dev = "cuda" if dist.get_backend() == "nccl" else "cpu"
        mine = torch.frombuffer(bytearray(blob), dtype=torch.uint8).to(dev)
        allp = torch.empty(world * mine.numel(), dtype=torch.uint8, device=dev)
        dist.all_gather_into_tensor(allp, mine)
        raw = allp.cpu().numpy().tobytes()
        blobs = [raw[r * mine.numel():(r + 1) * mine.numel()] for r in range(world)]
        got = xpl.combine_partials(blobs, 50, 0, 256)
        ms.append((time.perf_counter() - t0) * 1e3)
    ctx.close()
    dt = _allmax(torch, dist, min(ms))
    out = {"words": words, "ranks": world, "ms": dt, "gbs": words / (dt / 1e3) / 1e9,
           "note": "reset=0 (1 B/word); wall-clock of partial diagnose + all_gather + combine, max over ranks"}
    if rank == 0 and check_1gpu:
        ref = xpl.Context(pool_words=words + (1 << 16), max_rows=16)
        ref.register(base, 4 * words, xpl.ALLOC_DEVICE)
        ref.record_copy(base, 0x1000, 2 * words, xpl.COPY_H2D)
        ref.kernel_begin(s)
        ref.touch(base, words, 7, s, 0)
        ref.kernel_end(s)
        exp = ref.diagnose(50, 0, 256, reset=False)
        ref.close()
        out["identical_to_unsharded"] = exp == got
    return out


def _allmax(torch, dist, x):
    if not dist.is_available() or not dist.is_initialized():
        return x
    dev = "cuda" if dist.get_backend() == "nccl" else "cpu"
    t = torch.tensor([x], dtype=torch.float64, device=dev)
    dist.all_reduce(t, op=dist.ReduceOp.MAX)
    return float(t.item())


def atomic_peaks(xpl, torch, reps=3):
    """The recording roofline's denominator: 32-bit atomic OR
    throughput of this B200 from the in-repo microbenchmark, one op per distinct
    u32, coalesced: RED (what a hook's commit issues) and ATOM over 1 GiB (HBM
    backed) and over 32 MiB (L2 resident), plus the same-u32-per-warp case."""
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


def diag_at_scale(xpl, torch, words=1 << 31, reps=3):
    """The diagnose pass over a cfg5-sized shadow (2^31 words = 2 GiB, SURVEY §8(d)
    cfg5 ~2.2e9 words) with a mixed realistic content: CPU-written half (H2D),
    GPU reads/writes in 4096-word blocks and random regions.  Timed live with
    CUDA events on the runtime stream (xpl_profile)."""
    ctx = xpl.Context(pool_words=words + (1 << 16), max_rows=16)
    base = 1 << 44  # synthetic address range: hooks only use addresses
    ctx.register(base, 4 * words, xpl.ALLOC_DEVICE)
    ctx.record_copy(base, 0x1000, 2 * words, xpl.COPY_H2D)
    st = torch.cuda.current_stream()
    s = st.cuda_stream
    ctx.sync()
    torch.cuda.synchronize()
    # recording at scale: the synthetic instrumented kernel's hooks + the epoch close
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
    # shadow u32s the hooks committed to: one RED each (first touch, warp-aggregated)
    import numpy as np
    n_red = 0
    for w0 in range(0, words, 1 << 28):
        d = ctx.shadow_dump(base, w0, min(1 << 28, words - w0)).view(np.uint32)
        n_red += int(np.count_nonzero(d & 0xC8C8C8C8))
    for _ in range(reps):
        ctx.diagnose(50, 0, 256, reset=False)
    p0 = ctx.profile_read(reset=True)
    # the UM page view (NEXT-3) over the same shadow: one read pass; blocking
    # call, timed whole (host wall clock around it, device work dominates)
    import time
    ctx.page_summary(1024)
    pv = []
    for _ in range(reps):
        t0 = time.perf_counter()
        ctx.page_summary(1024)
        pv.append((time.perf_counter() - t0) * 1e3)
    pv_ms = min(pv)
    rep = ctx.diagnose(50, 0, 256, reset=True)
    p1 = ctx.profile_read(reset=True)
    ctx.profile(False)
    ctx.close()
    n_dev = rep[0]["gpu_acc"]  # each word is hooked at most once by the touch kernel
    out = {"record": {"device_accesses": n_dev, "ms": rec_ms, "accesses_per_s": n_dev / (rec_ms / 1e3),
                      "fold_ms": pf["ms"], "fold_gbs": pf["bytes"] / (pf["ms"] / 1e3) / 1e9 if pf["ms"] else None,
                      "shadow_u32_committed": n_red,
                      "note": "instrumented touch kernel (hooks only, no user data) + epoch close, events on its stream"},
           "page_view": {"words": words, "page_words": 1024, "whole_call_ms": pv_ms,
                         "kernel_ms": p1["pages"]["ms"] / max(1, p1["pages"]["launches"]),
                         "gbs": (p1["pages"]["bytes"] / (p1["pages"]["ms"] / 1e3) / 1e9) if p1["pages"]["ms"] else None,
                         "note": "xpl_page_summary's page_kernel (1 B per word read), CUDA events, mean of 4 calls"}}
    for name, p in (("no_reset", p0), ("reset", p1)):  # (the loop below fills these two)
        d = p["diag_tile"]
        ms = d["ms"] / d["launches"]
        out[name] = {"words": words, "ms": ms, "gbs": d["bytes"] / d["launches"] / (ms / 1e3) / 1e9,
                     "bytes_per_launch": d["bytes"] / d["launches"],
                     "whole_call_ms": p["diagnose"]["ms"] / p["diagnose"]["launches"]}
    return out


def other_configs(xpl, apps, torch, lulesh_steps=100, lulesh250_steps=10):
    """The other BASELINE.json configs, each run once instrumented and once as the
    uninstrumented twin, device-timed: cfg1 SW-128 (one cooperative launch, 4
    epochs), cfg3 SW-16K (32,767 per-diagonal epochs, host traceback segments and
    diagnoses every 1,024 diagonals), cfg4 LULESH-shaped 100^3 x 100 timesteps,
    cfg5 LULESH-shaped 250^3 (1.47e9 + 0.84e9 shadow words per timestep) on one
    GPU for 10 timesteps (the 100-timestep run is 10x this; its shadow fits one
    B200)."""
    from xplgen import lulesh as L
    from xplgen import sw
    out = {}
    us = torch.cuda.Stream()

    def timed_run(ctx, fn):
        s = torch.cuda.ExternalStream(ctx.runtime_stream()) if ctx is not None else us
        torch.cuda.synchronize()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record(s)
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
            for c in (ctx, None):
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
    for name, s_edge, steps, pool in (("cfg4_lulesh100", 100, lulesh_steps, 1 << 28),
                                      ("cfg5_lulesh250", 250, lulesh250_steps, 2_500_000_000)):
        if not steps:
            continue
        spec = L.lulesh_spec(s_edge)
        ar = apps.Arena(spec)
        topo = L.topology(s_edge, 0x58504C05)
        hc = torch.zeros(1, dtype=torch.int64, device="cuda")
        res = {}
        with xpl.Context(pool_words=pool, max_rows=64) as ctx:
            for c in (ctx, None):
                apps.lulesh_prepare(ar, s_edge, topo)
                hc.zero_()

                def fn(c):
                    run = apps.Run(c, us.cuda_stream, params=PARAMS, out_cap=64 * (steps + 1))
                    apps.lulesh(run, ar, s_edge, steps, hc)
                    return run
                ms, run = timed_run(c, fn)
                res["instr" if c is not None else "twin"] = (ms, int(hc.item()) + run.r.host_accesses,
                                                            run.r.epochs, run.r.n_diag, run.r.host_ms)
        del ar, topo
        acc = res["instr"][1]
        out[name] = {"workload": f"LULESH-shaped {s_edge}^3 x {steps} timesteps, 50 managed "
                                 "allocations + 2 temporaries/step, 19 launches/step",
                     "ms": res["instr"][0], "accesses": acc,
                     "accesses_per_s": acc / (res["instr"][0] / 1e3), "epochs": res["instr"][2],
                     "diagnoses": res["instr"][3], "host_ms": res["instr"][4],
                     "twin_ms": res["twin"][0], "slowdown": res["instr"][0] / res["twin"][0]}
    return out


def reference_main(args):
    rank = int(os.environ.get("RANK", "0"))
    if rank != 0:
        return
    for _ in range(args.warmup):  # untimed warm-up samples (short)
        cpu_baseline(seconds_budget=1.0)
    steps = []
    for _ in range(max(1, args.steps)):
        steps.append(cpu_baseline())
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
    backend = os.environ.get("XPL_DIST_BACKEND", "nccl")  # gloo: test the N>1 logic on one GPU
    if world > 1:
        if backend == "nccl":
            dist.init_process_group("nccl", device_id=torch.device("cuda", local))
        else:
            dist.init_process_group(backend)

    from paper_conf_ipps_pirkelbauerlvl20_b200 import apps, xpl
    from xplgen import rodinia

    ctx = xpl.Context(device=local, pool_words=1 << 27, max_rows=256)
    rs = torch.cuda.ExternalStream(ctx.runtime_stream())
    us = torch.cuda.Stream()
    hs = rodinia.hotspot_spec(HOT[0], HOT[1])
    bs = rodinia.backprop_spec(*BACKPROP)
    fs = rodinia.bfs_spec(*BFS)
    ns = rodinia.nw_spec(NW[0])
    ar_h, ar_b, ar_f, ar_n = apps.Arena(hs), apps.Arena(bs), apps.Arena(fs), apps.Arena(ns)
    rodinia.fill_inputs("hotspot", ar_h.host_views(), 0x58504C01)
    rodinia.fill_inputs("backprop", ar_b.host_views(), 0x58504C01)
    edges = rodinia.bfs_graph(BFS[0], BFS[1], 0x58504C02)
    nw_in = rodinia.nw_inputs(NW[0], NW[1], 0x58504C03)
    hook_ctr = torch.zeros(1, dtype=torch.int64, device="cuda")
    flush_buf = torch.empty(256 << 20, dtype=torch.uint8, device="cuda")  # > 126 MB L2
    levels = [0]

    def prepare(do_copies):
        """Untimed: the programs' inputs (bfs graph + resident device state, nw sequences)."""
        apps.bfs_prepare(ar_f, BFS[0], BFS[1], edges, resident=not do_copies)
        rodinia.nw_fill_host(ar_n.host_views(), ns, nw_in, NW[0])
        hook_ctr.zero_()

    def step(c, do_copies, time_kernels=False):
        counts = [0, 0, 0, 0, 0.0, 0.0]
        progs = ((apps.hotspot, ar_h, HOT), (apps.backprop, ar_b, BACKPROP),
                 (apps.bfs, ar_f, BFS + (hook_ctr,)), (apps.nw, ar_n, NW + (nw_in["blosum"],)))
        for fn, ar, a in progs:
            run = apps.Run(c, us.cuda_stream, do_copies=do_copies, diag_each=True, params=PARAMS,
                           time_kernels=time_kernels)
            r = fn(run, ar, *a)
            if fn is apps.bfs:
                levels[0] = r
            counts[0] += run.r.dev_accesses
            counts[1] += run.r.host_accesses
            counts[2] += run.r.copy_words
            counts[3] += run.r.epochs
            counts[4] += run.r.kernel_ms
            counts[5] += run.r.host_ms
        return counts

    def timed(c, do_copies, steps, stream):
        total, counts = 0.0, None
        for _ in range(steps):
            prepare(do_copies)
            flush_buf.random_(0, 255)  # flush L2 between steps (untimed)
            torch.cuda.synchronize()
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            e0.record(stream)
            counts = step(c, do_copies)
            if c is not None:
                c.join(stream.cuda_stream)  # the runtime's last work may sit on the user stream
            e1.record(stream)
            e1.synchronize()
            us.synchronize()
            total += e0.elapsed_time(e1)
            if c is not None:
                counts[0] += int(hook_ctr.item())  # bfs hook calls (data dependent)
                hook_ctr.zero_()
        return total, counts

    clk = Clocks(local)  # sampler up before the warm-up; clk.mark() opens the timed window
    for _ in range(args.warmup):
        prepare(False)
        step(ctx, False)
    torch.cuda.synchronize()

    # --- value: device-timed, app data resident -------------------------------
    # (no per-kernel events here: they cost 4-8 ms per step -- they break the
    # fold's programmatic launch behind each epoch -- profiles/r1s_profiling_ab.txt)
    st0 = ctx.stats()
    if world > 1:
        dist.barrier()
    torch.cuda.synchronize()
    clk.mark()
    ms_total, counts = timed(ctx, False, args.steps, rs)
    clocks = clk.stop()
    st1 = ctx.stats()
    per_step = counts[0] + counts[1] + counts[2]
    ms_max = _allmax(torch, dist, ms_total)
    value = per_step * args.steps * world / (ms_max / 1e3)
    launches = (st1["kernel_launches"] - st0["kernel_launches"]) + counts[3] * args.steps

    # --- the same K steps again, every runtime kernel bracketed by CUDA events on
    # its stream (xpl_profile): the roofline's launch durations -------------------
    ctx.profile(True)
    if world > 1:
        dist.barrier()
    torch.cuda.synchronize()
    ms_prof, _ = timed(ctx, False, args.steps, rs)
    prof = ctx.profile_read(reset=True)
    ctx.profile(False)
    if args.step_only:
        ctx.close()
        return

    # --- e2e: with the programs' real copies -----------------------------------
    prepare(True)
    step(ctx, True)
    st0 = ctx.stats()
    if world > 1:
        dist.barrier()
    e2e_ms, _ = timed(ctx, True, args.steps, rs)
    st1 = ctx.stats()
    e2e_ms = _allmax(torch, dist, e2e_ms)
    rec_bytes = 8 * (st1["host_records_packed"] - st0["host_records_packed"]) // args.steps
    nwc = (NW[0] + 1) ** 2
    app_h2d = (4 * (2 * HOT[0] * HOT[1]) + 4 * ((BACKPROP[0] + 1) * (1 + 2 * (BACKPROP[1] + 1)) + BACKPROP[1] + 1)
               + (8 + 4 * BFS[1] + 3 + 4) * BFS[0] + levels[0] + 2 * 4 * nwc)
    app_d2h = (4 * HOT[0] * HOT[1] + 4 * ((BACKPROP[0] + 1) * (BACKPROP[1] + 2) + (BACKPROP[0] // 16) * BACKPROP[1])
               + 4 * BFS[0] + levels[0] + 4 * nwc)
    n_diag_rows = (HOT[2] + 1) * 6 + 11 + (levels[0] + 1) * 14 + 5  # report rows per step
    e2e = {"value": per_step * args.steps * world / (e2e_ms / 1e3), "unit": "accesses/s",
           "h2d_bytes_per_step": rec_bytes + app_h2d,
           "d2h_bytes_per_step": app_d2h + 208 * n_diag_rows}

    # --- uninstrumented twins (slowdown, Table III context) ------------------
    prepare(False)
    step(None, False)
    twin_ms, _ = timed(None, False, args.steps, us)

    # --- breakdown (untimed pass with per-kernel events) ----------------------
    prepare(False)
    bi = step(ctx, False, time_kernels=True)
    prepare(False)
    bt = step(None, False, time_kernels=True)
    torch.cuda.synchronize()

    # --- launch log of one untimed step (NEXT-4): per kernel, its epochs' GPU
    # time (incl. fold) and write footprint, measured in stream order ----------
    prepare(False)
    ctx.launch_log_enable(True)
    step(ctx, False)
    llog = ctx.launch_log(reset=True)
    ctx.launch_log_enable(False)
    launch_log = {}
    for r in llog:
        k = launch_log.setdefault(r["name"], {"launches": 0, "epoch_ms_sum": 0.0, "written_chunks": 0,
                                              "grid_example": r["grid"], "block": r["block"]})
        k["launches"] += 1
        k["epoch_ms_sum"] += r["epoch_ms"] / max(1, r["launches_in_epoch"])
        k["written_chunks"] += r["epoch_written_chunks"] // max(1, r["launches_in_epoch"])

    # --- the diagnose pass at cfg5 scale; the other configs -------------------
    at_scale = diag_at_scale(xpl, torch)
    atom = atomic_peaks(xpl, torch)
    rec = at_scale["record"]
    rec["atomic_microbench"] = atom
    # recording roofline: accesses/s <= min(HBM / shadow bytes per
    # access, RED rate x accesses per RED); the touch kernel hooks each word once
    apr = rec["device_accesses"] / max(1, rec["shadow_u32_committed"])
    pk, _ = peaks()
    rec["reds_per_s"] = rec["shadow_u32_committed"] / (rec["ms"] / 1e3)
    rec["roofline_accesses_per_s"] = min(pk * 1e9 / 2.0, atom["red_hbm_per_s"] * apr)
    rec["frac"] = rec["accesses_per_s"] / rec["roofline_accesses_per_s"]
    sharded = None
    if world > 1:
        try:
            sharded = diag_sharded(xpl, torch, dist, rank, world)
        except Exception as ex:  # keep the primary line even if this extra fails
            sharded = {"error": repr(ex)}
    others = other_configs(xpl, apps, torch) if not args.no_other_configs else None

    # --- roofline of the dominant runtime kernel -------------------------------
    peak, peak_src = peaks()
    dom = max(("diag_tile", "merge", "range", "fold"), key=lambda k: prof[k]["ms"])
    d = prof[dom]
    achieved = (d["bytes"] / d["launches"]) / (d["ms"] / d["launches"] / 1e3) / 1e9 if d["launches"] else 0.0
    traffic = None  # DRAM bytes per launch of that kernel from an ncu capture (profiles/traffic.json)
    try:
        tj = json.load(open(os.path.join(os.path.dirname(os.path.abspath(__file__)), "profiles", "traffic.json")))
        traffic = tj[dom]["bytes_per_launch"] if dom in tj else None
    except (OSError, ValueError, KeyError):
        pass
    roof = {"kernel": dom, "bound": "hbm", "achieved": achieved, "peak": peak, "unit": "GB/s",
            "frac": achieved / peak, "traffic": traffic, "peak_source": peak_src,
            "algorithmic_bytes_per_launch": d["bytes"] / max(1, d["launches"]),
            "avg_launch_ms": d["ms"] / max(1, d["launches"]),
            "share_of_step": d["ms"] / ms_prof,
            "timing": "launch durations from a second, profiled run of the same K steps (events on the kernel's stream); value from the unprofiled run"}
    dg = prof["diag_tile"]
    line = {
        "metric": METRIC,
        "value": value, "unit": "accesses/s", "n_gpus": world, "steps": args.steps, "warmup": args.warmup,
        "ms_per_step": ms_max / args.steps, "higher_is_better": True, "scaling": "weak",
        "vs_baseline": None, "dtype": "u8", "data": "synthetic",
        "config": {"workload": WORKLOAD, "accesses_per_step": per_step, "device_accesses": counts[0],
                   "host_accesses": counts[1], "transfer_words": counts[2], "epochs_per_step": counts[3],
                   "diag_params": {"threshold_pct": PARAMS[0], "block_words": PARAMS[1], "min_run": PARAMS[2]},
                   "l2": "flushed between steps (256 MB write, untimed)", "parallelism": f"replicas x{world}"},
        "roofline": roof,
        "diagnose_gbs": at_scale["reset"]["gbs"],
        "diagnose_at_scale": dict(at_scale, peak_gbs=peak, frac_reset=at_scale["reset"]["gbs"] / peak,
                                  frac_no_reset=at_scale["no_reset"]["gbs"] / peak),
        "diagnose_gbs_in_step": (dg["bytes"] / (dg["ms"] / 1e3) / 1e9) if dg["ms"] else None,
        "profiled_ms_per_step": ms_prof / args.steps,
        "runtime_kernels": {k: {"launches": v["launches"], "ms_per_step": v["ms"] / args.steps,
                                "gbs": (v["bytes"] / (v["ms"] / 1e3) / 1e9) if v["ms"] else None}
                            for k, v in prof.items()},
        "breakdown_ms_per_step": {"instrumented_kernels": bi[4], "twin_kernels": bt[4],
                                  "host_tracer": bi[5],
                                  "runtime_kernels": sum(v["ms"] for k, v in prof.items() if k != "diagnose" and k != "diag_tile") / args.steps + prof["diagnose"]["ms"] / args.steps},
        "slowdown": {"kernels_only": bi[4] / bt[4] if bt[4] else None,
                     "whole_program": (ms_total / args.steps) / (twin_ms / args.steps),
                     "twin_ms_per_step": twin_ms / args.steps,
                     "paper_context": "Table III P:L431-443: 5x-20x, avg ~15x (Intel E5-2695 v4 + Pascal, CUDA 9.2)"},
        "e2e": e2e, "gpu_launches": int(launches), "clocks": clocks,
        "launch_log": launch_log,
        "other_configs": others,
        "diagnose_sharded": sharded,
    }
    if rank == 0 and world == 1 and not args.no_cpu_baseline:
        line["cpu_baseline"] = cpu_baseline()
    if rank == 0:
        print(json.dumps(line), flush=True)
    ctx.close()
    if world > 1:
        dist.destroy_process_group()


if __name__ == "__main__":
    main()

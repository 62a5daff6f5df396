#!/usr/bin/env python
"""Expected reports of the full-size configs, computed by the ORACLE ONLY.

TEST INFRASTRUCTURE (like oracle/): writes tests/golden/fullsize/<cfg>.json,
which tests/test_gpu_fullsize_cfg34.py compares the CUDA path's full-size runs
with.  Nothing here touches the CUDA path: the events are the CPU twins of the
workload programs (xplgen), replayed by oracle/xpl_oracle.cpp.

The full-size traces (cfg3 ~2.1e9 events, cfg4 ~4e8 per timestep) take the
oracle tens of minutes on one core, too long for a test, so the expected
reports are computed once here (the oracle is deterministic; the workloads are
seeded) and stored.  Two transformations keep the replay inside memory and
time; both leave every per-word record unchanged by definition, and
tests/test_golden_fullsize_cpu.py checks that on small sizes:
  * a device batch (one GPU epoch) is reduced to its distinct (word address,
    kind) events -- within an epoch multiplicity and order do not matter
    (snapshot semantics D5, counting D21);
  * a host batch is cut into maximal runs of consecutive, abutting accesses of
    one kind, each replayed as one range access (reading D28: equal to the
    per-access events when no access straddles two allocations, true here).
Allocation bases are synthetic; reports are compared without `base`.

  python tools/golden_fullsize.py cfg3|cfg4 [--out DIR]
  python tools/golden_fullsize.py cfg5 [--workers N]     (partitioned, then merged)

cfg5 (LULESH-shaped 250^3, 1.47e9 persistent + 0.84e9 temporary shadow words;
timesteps 1 and 2 + the final diagnose: the program is periodic from timestep 2
on, tests/test_golden_fullsize_cpu.py) does not fit one oracle process (a std::map node per word), so it is replayed
partitioned by allocation: each part replays the sampled twin
(xplgen.lulesh windows mode: every event of `dom`, `dt_block` and of the
part's arrays, nothing else -- a word's record depends only on the events that
touch it, D30) and keeps its arrays' rows; the force temporary (7.5e8 words) is
cut into word windows, whose rows are summed (it is never host-accessed, so
its transfer runs are zero in every window -- asserted -- and its density is
recomputed from the summed GPU words by Eq. P:L102 with whole-allocation
blocks, D11-D13).
"""
from __future__ import annotations

import argparse
import json
import os
import sys
import time

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

PARAMS = (50, 0, 256)  # bench.py PARAMS: threshold 50 %, whole-allocation blocks, min run 256
CFG4_STEPS = 3          # timesteps replayed in full (periodic after timestep 2)


def dedupe_device(op):
    a = np.asarray(op[1], np.uint64)
    z = np.asarray(op[2], np.uint64)
    k = np.asarray(op[3], np.uint64)
    assert a.max(initial=0) < (1 << 56) and z.max(initial=0) < 16
    key = np.unique((a << np.uint64(6)) | (z << np.uint64(2)) | k)  # size in bits 2-5, kind in 0-1
    return ("DB", key >> np.uint64(6), ((key >> np.uint64(2)) & np.uint64(15)).astype(np.uint32),
            (key & np.uint64(3)).astype(np.uint8))


def host_ranges(op):
    """Maximal runs of abutting accesses of one kind, in program order."""
    a = np.asarray(op[1], np.uint64)
    z = np.asarray(op[2], np.uint64)
    k = np.asarray(op[3], np.uint8)
    if a.size == 0:
        return
    brk = np.nonzero((a[1:] != a[:-1] + z[:-1]) | (k[1:] != k[:-1]))[0] + 1
    starts = np.concatenate([[0], brk])
    ends = np.concatenate([brk, [a.size]])
    for s, e in zip(starts.tolist(), ends.tolist()):
        lo = int(a[s])
        hi = int(a[e - 1]) + int(z[e - 1])
        yield ("H", lo, hi - lo, int(k[s]))


def reduced(ops):
    """The two record-preserving transformations (module docstring)."""
    for op in ops:
        if op[0] == "DB":
            yield dedupe_device(op)
        elif op[0] == "HB":
            yield from host_ranges(op)
        else:
            yield op


def replay(ops, log=None):
    from oracle import Oracle
    o = Oracle()
    out, t0, n = [], time.time(), 0
    for op in ops:
        if op[0] in ("DB", "HB"):
            n += len(op[1])
        r = o.op(op)
        if r is not None:
            out.append([{f: v for f, v in row.items() if f != "base"} for row in r])
            if log:
                log(f"diag {len(out)}: {time.time() - t0:.0f} s, {n} events")
    o.close()
    return out


def cfg3_ops():
    from xplgen import sw
    from xplgen.rodinia import layout
    n = m = 16384
    spec = sw.sw_spec(n, m)
    addrs, _, _ = layout(spec, 0, 0, 1 << 40)
    inp = sw.sw_inputs(n, m, 0x58504C04)  # bench.py other_configs: the cfg3 program's inputs
    meta = {"config": "cfg3 Smith-Waterman 16384x16384, per-diagonal launches, traceback reads and a "
                      "diagnose every 1024 diagonals", "n": n, "m": m, "per_diagonal": 1, "tb_every": 1024,
            "diag_every": 1024, "seed": 0x58504C04, "params": PARAMS}
    return sw.sw_trace_iter(addrs, spec, n, m, 1, 1024, 1024, inp, PARAMS), meta


def cfg4_ops(s=100, steps=CFG4_STEPS):
    from xplgen import lulesh as L
    from xplgen.rodinia import layout
    spec = L.lulesh_spec(s)
    addrs, _, _ = layout(spec, 0, 0, 1 << 40)
    topo = L.topology(s, 0x58504C05)
    tmps = [((1 << 44) + t * (1 << 34), (1 << 44) + t * (1 << 34) + (1 << 33)) for t in range(steps)]
    meta = {"config": f"cfg4 LULESH-shaped {s}^3, first {steps} timesteps + final frees/diagnose "
                      "(reset every timestep)", "s": s, "steps": steps, "seed": 0x58504C05, "params": PARAMS}
    return L.lulesh_trace_iter(addrs, spec, s, steps, topo, PARAMS, tmps), meta


CFG5_STEPS = 2  # timestep 1 (after the host init) and timestep 2 (steady state: periodic from here on)
CFG5_GROUPS = [  # array slots per part (<= ~1.3e8 words each)
    (0, 1, 2, 3), (4, 5, 6, 7), (8, 9, 10, 11), (12, 27, 28, 31, 32, 37, 38),
    (13, 14, 15, 16), (17, 18, 19, 20), (21, 22, 23, 24), (25, 29, 33, 34), (35, 36, 39, 40),
    (41, 42, 43, 44), (45, 46, 47), (26,), (30,)]
CFG5_TMP_WINDOWS = 6  # the force temporary in windows of 1.25e8 words


def cfg5_ops(slots=(), tmp=None, s=250, steps=CFG5_STEPS):
    from xplgen import lulesh as L
    from xplgen.rodinia import layout
    spec = L.lulesh_spec(s)
    addrs, _, _ = layout(spec, 0, 0, 1 << 40)
    topo = L.topology(s, 0x58504C05)
    tmps = [((1 << 44) + t * (1 << 36), (1 << 44) + t * (1 << 36) + (1 << 35)) for t in range(steps)]
    win = {k: [(0, L.slot_bytes(s, k) // 4)] for k in slots}
    return L.lulesh_trace_iter(addrs, spec, s, steps, topo, PARAMS, tmps, windows=win, reset=1, final=True,
                               tmp_windows=tmp)


def cfg5_part(name, slots, tmp, out):
    """One part: the reports' rows of `slots` (ids 2 + k), of dom / dt_block
    (ids 0, 1), and of the temporaries (ids >= 50) when tmp windows are given."""
    keep = {0, 1} | {2 + k for k in slots}
    t0 = time.time()
    diags = replay(reduced(cfg5_ops(slots, tmp)))
    rows = [[r for r in d if r["id"] in keep or (tmp and r["id"] >= 50)] for d in diags]
    with open(out, "w") as f:
        json.dump({"name": name, "slots": list(slots), "tmp": tmp, "seconds": round(time.time() - t0, 1),
                   "diagnoses": rows}, f)


def cfg5_merge(parts, s=250):
    """Rows by id; the force temporary's windows summed (module docstring)."""
    from xplgen import lulesh as L
    thr = PARAMS[0]
    n = len(parts[0]["diagnoses"])
    out = []
    for d in range(n):
        rows, tmp = {}, {}
        for p in parts:
            for r in p["diagnoses"][d]:
                if r["id"] >= 50 and p["tmp"]:
                    tmp.setdefault(r["id"], []).append(r)
                else:
                    rows[r["id"]] = r
        for i, rs in tmp.items():
            o = dict(rs[0])
            for f in ("w_c", "w_g", "r_cc", "r_cg", "r_gc", "r_gg", "any_acc", "gpu_acc", "alternating"):
                o[f] = sum(r[f] for r in rs)
            for r in rs:
                assert r["h2d_unused_runs"] == r["d2h_unneeded_runs"] == r["w_c"] == 0 and r["r_cc"] == r["r_gc"] == 0
            o["ever_accessed"] = max(r["ever_accessed"] for r in rs)
            o["density_pct_any"] = o["any_acc"] * 100 // o["words"]
            o["density_pct_gpu"] = o["gpu_acc"] * 100 // o["words"]
            f = o["gpu_acc"] >= 1 and 100 * o["gpu_acc"] <= thr * o["words"]
            o["low_density_blocks"], o["low_density_words"] = (1, o["words"]) if f else (0, 0)
            o["flags"] = (1 if o["alternating"] else 0) | (2 if f else 0) | (16 if o["any_acc"] == 0 else 0)
            rows[i] = o
        out.append([rows[k] for k in sorted(rows)])
    return out


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("cfg", choices=["cfg3", "cfg4", "cfg5", "cfg5-part"])
    ap.add_argument("--out", default=os.path.join(ROOT, "tests", "golden", "fullsize"))
    ap.add_argument("--workers", type=int, default=3)
    ap.add_argument("--part", type=int, default=-1)
    ap.add_argument("--no-merge", action="store_true")
    ap.add_argument("--only", default="", help="cfg5: comma-separated part names to run (default: all missing)")
    a = ap.parse_args()
    if a.cfg in ("cfg5", "cfg5-part"):
        from xplgen import lulesh as L
        jobs = [(f"g{i}", g, None) for i, g in enumerate(CFG5_GROUPS)]
        fw = 24 * 250 ** 3 * 2
        step = (-(-fw // CFG5_TMP_WINDOWS) + 1) & ~1  # (windows cut between 8-byte elements)
        jobs += [(f"force{i}", (), {0: [(i * step, min(fw, (i + 1) * step))]}) for i in range(CFG5_TMP_WINDOWS)]
        jobs.append(("dvdx", (), {1: [(0, 3 * 250 ** 3 * 2)]}))
        pdir = os.path.join(a.out, "cfg5_parts")
        os.makedirs(pdir, exist_ok=True)
        if a.cfg == "cfg5-part":
            name, slots, tmp = jobs[a.part]
            cfg5_part(name, slots, tmp, os.path.join(pdir, name + ".json"))
            return
        import subprocess
        only = set(filter(None, a.only.split(",")))
        todo = [i for i, j in enumerate(jobs) if not os.path.exists(os.path.join(pdir, j[0] + ".json"))
                and (not only or j[0] in only)]
        todo.sort(key=lambda i: -(sum(L.slot_bytes(250, k) for k in jobs[i][1]) + (1 << 40 if jobs[i][2] else 0)))
        running = []
        while todo or running:
            while todo and len(running) < a.workers:
                i = todo.pop(0)
                running.append(subprocess.Popen([sys.executable, __file__, "cfg5-part", "--part", str(i),
                                                 "--out", a.out]))
            time.sleep(5)
            for p in list(running):
                if p.poll() is not None:
                    if p.returncode != 0:
                        print("part failed:", p.args, p.returncode, flush=True)
                    running.remove(p)
            print(f"{len(todo)} to do, {len(running)} running", flush=True)
        if a.no_merge:
            return
        parts = [json.load(open(os.path.join(pdir, j[0] + ".json"))) for j in jobs]
        meta = {"config": f"cfg5 LULESH-shaped 250^3, first {CFG5_STEPS} timesteps + final frees/diagnose "
                          "(reset every timestep), partitioned by allocation", "s": 250, "steps": CFG5_STEPS,
                "seed": 0x58504C05, "params": PARAMS, "parts": [p["name"] for p in parts],
                "oracle_seconds": sum(p["seconds"] for p in parts),
                "written_by": "tools/golden_fullsize.py cfg5 (oracle/ only)"}
        with open(os.path.join(a.out, "cfg5.json"), "w") as f:
            json.dump({"meta": meta, "diagnoses": cfg5_merge(parts)}, f)
        print("wrote cfg5")
        return
    ops, meta = cfg3_ops() if a.cfg == "cfg3" else cfg4_ops()
    t0 = time.time()
    diags = replay(reduced(ops), log=lambda s: print(s, flush=True))
    meta["oracle_seconds"] = round(time.time() - t0, 1)
    meta["written_by"] = "tools/golden_fullsize.py (oracle/ only)"
    os.makedirs(a.out, exist_ok=True)
    with open(os.path.join(a.out, a.cfg + ".json"), "w") as f:
        json.dump({"meta": meta, "diagnoses": diags}, f)
    print("wrote", a.cfg, len(diags), "diagnoses in", meta["oracle_seconds"], "s")


if __name__ == "__main__":
    main()

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


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("cfg", choices=["cfg3", "cfg4"])
    ap.add_argument("--out", default=os.path.join(ROOT, "tests", "golden", "fullsize"))
    a = ap.parse_args()
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
